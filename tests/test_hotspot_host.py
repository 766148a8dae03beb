"""Host-side tests of the HotSpot-2D path (NEXT-3) without a GPU: the
planner's op lists (blocks + borders moved down, leaf launches on shrinking
windows, blocks moved up, passes alternating grids) replayed on the CPU with
the oracle's window update in ANY dependency-respecting order reproduce the
oracle's plain sweep bit for bit (fp64), across siblings too; byte counts and
capacities follow the plan's closed forms."""
import random

import numpy as np
import pytest

import nugen
import paper_conf_ipps_chey19_b200 as nu
from oracle import hotspot as hs

K = hs.coeffs(1024, 1024)


def grids(R, C, seed):
    return (nugen.fill(R, C, seed, nugen.MAT_T, "temp"), nugen.fill(R, C, seed, nugen.MAT_P, "power"))


def simulate_hotspot(plan, T, P, R, C, rng=None):
    bufs, ops = plan.bufs(), plan.ops()
    mem = []
    for b in bufs:
        if b["kind"] == 0:
            mem.append(T.astype(np.float64).ravel().copy())
        elif b["kind"] == 1:
            mem.append(P.astype(np.float64).ravel().copy())
        else:
            mem.append(np.full(max(b["bytes"] // 4, R * C if b["kind"] == 2 else 0), np.nan))

    def view(buf, off, ld, rows, cols):
        return np.lib.stride_tricks.as_strided(mem[buf][off:], shape=(rows, cols),
                                               strides=(ld * 8, 8), writeable=True)

    def run(op):
        if op["op"] == nu.NU_OP_COPY:
            view(op["dst_buf"], op["dst_off"], op["dst_ld"], op["rows"], op["cols"])[...] = \
                view(op["src_buf"], op["src_off"], op["src_ld"], op["rows"], op["cols"]).copy()
            return
        assert op["op"] == nu.NU_OP_STENCIL
        m, n, it = op["m"], op["n"], op["k"]
        gy0, gx0, RR, CC = op["src_off"], op["dst_off"], op["rows"], op["cols"]
        cur = view(op["a_buf"], op["a_off"], op["lda"], m, n).copy()
        p = view(op["b_buf"], op["b_off"], op["ldb"], m, n).copy()
        for _ in range(it):
            cur = hs._window_step(cur, p, gy0, gx0, RR, CC, K)
        vy0 = 0 if gy0 == 0 else it
        vy1 = m if gy0 + m == RR else m - it
        vx0 = 0 if gx0 == 0 else it
        vx1 = n if gx0 + n == CC else n - it
        assert not np.isnan(cur[vy0:vy1, vx0:vx1]).any(), "leaf read a cell that was never loaded"
        view(op["c_buf"], op["c_off"], op["ldc"], m, n)[vy0:vy1, vx0:vx1] = cur[vy0:vy1, vx0:vx1]

    if rng is None:
        for op in ops:
            run(op)
    else:
        queues = {}
        for i, op in enumerate(ops):
            queues.setdefault((op["worker"], op["stream"]), []).append(i)
        done = set()
        while len(done) < len(ops):
            ready = [q for q in queues.values() if q and all(d in done for d in ops[q[0]]["deps"])]
            assert ready, "deadlock"
            i = rng.choice(ready).pop(0)
            run(ops[i])
            done.add(i)
    return mem[[b["kind"] for b in bufs].index(2)][: R * C].reshape(R, C)


@pytest.mark.parametrize("R,C,iters,G,cap,block,halo,leaf", [
    (40, 56, 6, 1, 0, 16, 3, 2),        # 2 passes, 2 launches per visit
    (33, 20, 5, 2, 0, 8, 0, 0),         # 2 siblings, automatic border (one pass)
    (64, 64, 9, 1, 0, 64, 4, 4),        # one block (window = grid), 3 passes
    (50, 30, 7, 3, 0, 12, 7, 8),        # 3 siblings, ragged blocks
    (70, 45, 11, 2, 0, 16, 2, 1),       # 6 passes (odd/even grid alternation), leaf_iters 1
    (96, 96, 10, 1, 200_000, 0, 5, 0),  # capacity picks the block
    (600, 520, 9, 2, 0, 300, 4, 4),     # 3 passes, 2 siblings: first / last blocks split 2 x 2
    (512, 512, 6, 1, 0, 256, 0, 0),     # one pass: its first and last blocks split
])
def test_hotspot_plan_replays_exactly(R, C, iters, G, cap, block, halo, leaf):
    T, P = grids(R, C, seed=R + C + iters)
    ref = hs.run(T, P, iters, K)
    t, _ = nu.host_tree(G, cap)
    p = t.hotspot_plan(R, C, iters, nu.hotspot_opts(block=block, halo=halo, leaf_iters=leaf))
    assert np.array_equal(simulate_hotspot(p, T, P, R, C), ref)
    for seed in range(3):
        out = simulate_hotspot(p, T, P, R, C, rng=random.Random(seed))
        assert np.array_equal(out, ref), f"order seed {seed} broke a dependency"
    s = p.stats()
    b, h = s["bm"], s["bk"]
    if b >= 256:   # split blocks: more windows than the plain b x b grid
        nwin = sum(1 for o in p.ops() if o["op"] == nu.NU_OP_COPY and o["stream"] == 0) // 2
        assert nwin > -(-R // b) * -(-C // b) * -(-iters // h)
    assert s["bytes_d2h"] == 4 * R * C * -(-iters // h)          # every pass writes the grid once
    # every window byte arrives once: over PCIe, or (power columns shared with the
    # sibling's previous window of the same rows) by a device copy from its slot
    bufs = p.bufs()
    into_arena = sum(4 * o["rows"] * o["cols"] for o in p.ops()
                     if o["op"] == nu.NU_OP_COPY and bufs[o["dst_buf"]]["kind"] == 3)
    assert s["bytes_h2d"] + s["bytes_d2d"] == into_arena
    if -(-C // b) > 1:
        assert s["bytes_d2d"] > 0
    if cap:
        assert all(x["bytes"] <= cap for x in p.bufs() if x["kind"] == 3)
    t.destroy()


def test_hotspot_in_hbm_plan():
    R, C, iters = 37, 29, 19
    T, P = grids(R, C, seed=3)
    t = nu.hbm_tree(0)
    p = t.hotspot_plan(R, C, iters)
    ops = p.ops()
    assert [o["op"] for o in ops] == [nu.NU_OP_STENCIL] * 3 and [o["k"] for o in ops] == [8, 8, 3]
    assert ops[-1]["c_buf"] == [b["kind"] for b in p.bufs()].index(2)      # the last launch writes Tout
    assert np.array_equal(simulate_hotspot(p, T, P, R, C), hs.run(T, P, iters, K))
    t.destroy()


def test_hotspot_default_coefficients_match_the_model():
    k = nu.hotspot_coeffs(32768, 32768)
    for name in ("cap_1", "rx_1", "ry_1", "rz_1", "amb"):
        assert getattr(k, name) == np.float32(K[name])


def test_hotspot_zero_iterations_is_a_copy():
    t, _ = nu.host_tree(1)
    p = t.hotspot_plan(10, 12, 0)
    T, P = grids(10, 12, seed=1)
    assert np.array_equal(simulate_hotspot(p, T, P, 10, 12), T.astype(np.float64))
    t.destroy()
