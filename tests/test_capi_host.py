"""Host-side tests of the C ABI (no GPU): the library loads and exports every
symbol include/northup.h declares; the tree (Listing 1) validates and
answers queries; the planner's op lists compute C = A.B exactly when replayed
by a CPU simulator in ANY order the dependencies allow (so the dependencies
are sufficient), move the closed-form number of bytes, and stay within node
capacities; the partitioner picks the grids of SURVEY.md §8(e)."""
import random

import numpy as np
import pytest

import nugen
import paper_conf_ipps_chey19_b200 as nu

GiB = 1 << 30


def test_library_exports_every_header_symbol():
    syms = nu.header_symbols()
    assert len(syms) >= 35
    L = nu.lib()
    missing = [s for s in syms if not hasattr(L, s)]
    assert not missing
    assert nu.version() == 100


def test_tree_queries_and_levels():
    t = nu.Tree()
    root = t.add_node(-1, nu.NU_HOST)
    h0 = t.add_node(root, nu.NU_HBM, 0, 8 * GiB)
    s0 = t.add_node(h0, nu.NU_SMEM, 0, 227 * 1024, nu.NU_PROC_SM100)
    h1 = t.add_node(root, nu.NU_HBM, 1, 8 * GiB, nu.NU_PROC_SM100)
    assert [t.get_level(n) for n in (root, h0, s0, h1)] == [0, 1, 2, 1]
    assert t.get_max_treelevel() == 2
    assert t.get_children_list(root) == [h0, h1]
    assert t.get_parent(s0) == h0 and t.get_parent(root) == -1
    assert t.fetch_node_type(h1) == nu.NU_HBM
    info = t.node_info(s0)
    assert info["is_leaf"] == 1 and info["processor_type"] == nu.NU_PROC_SM100
    txt = t.print()
    assert "HOST" in txt and "SMEM" in txt and "(leaf)" in txt and txt.count("\n") == 4
    t.destroy()


def test_tree_errors():
    t = nu.Tree()
    root = t.add_node(-1, nu.NU_HOST)
    with pytest.raises(nu.NorthupError) as e:
        t.add_node(-1, nu.NU_HOST)            # a second root
    assert e.value.code == nu.NU_EINVAL
    with pytest.raises(nu.NorthupError):
        t.add_node(17, nu.NU_HBM, 0)          # unknown parent
    with pytest.raises(nu.NorthupError):
        t.set_block(root, 64, 64, 30)         # bk not a multiple of 4
    h = t.add_node(root, nu.NU_HBM, 0)        # leaf without a processor
    with pytest.raises(nu.NorthupError) as e:
        t.finalize()
    assert e.value.code == nu.NU_EINVAL and "processor" in str(e.value)
    t.destroy()
    t = nu.Tree()
    h = t.add_node(-1, nu.NU_HBM, 0)
    t.add_node(h, nu.NU_HOST, -1, 0, nu.NU_PROC_SM100)   # edge to slower memory
    with pytest.raises(nu.NorthupError):
        t.finalize()
    t.destroy()


def test_gemm_needs_finalized_tree():
    t, _ = nu.host_tree(1)
    with pytest.raises(nu.NorthupError):
        nu.check(nu.lib().northup_gemm(t.handle, None, None, None, 4, 4, 4))
    t.destroy()


@pytest.mark.parametrize("G,M,N,grid", [(2, 65536, 65536, (2, 1)), (4, 65536, 65536, (2, 2)),
                                         (8, 65536, 65536, (4, 2)), (8, 1048576, 4096, (8, 1)),
                                         (1, 10, 10, (1, 1)), (3, 300, 900, (1, 3))])
def test_partition_grid(G, M, N, grid):
    assert nu.partition(G, M, N) == grid
    seen = np.zeros((M // 64 + 1, N // 64 + 1), dtype=int) if M * N > 1e6 else np.zeros((M, N), int)
    if M * N <= 1e6:
        for r in range(G):
            r0, r1, c0, c1 = nu.partition_region(G, M, N, 0, r)
            seen[r0:r1, c0:c1] += 1
        assert (seen == 1).all()


# ------------------------------------------------------------ plan simulator
def split_dead_mask(w_off, w_ld, w_rows, w_cols, so, sld, srows, sn):
    """Which values of a split region (off so, ld sld, srows x sn columns, split
    form: hi of column n at row element n/2, lo at sld/2 + n/2) a write of
    w_rows x w_cols at (w_off, w_ld) destroys."""
    dead = np.zeros((srows, sn), dtype=bool)
    if w_off + (w_rows - 1) * w_ld + w_cols <= so or so + srows * sld <= w_off:
        return dead
    n = np.arange(sn)
    for r in range(w_rows):
        a0, a1 = w_off + r * w_ld, w_off + r * w_ld + w_cols
        for sr in range(max(0, (a0 - so) // sld), min(srows, (a1 - 1 - so) // sld + 1)):
            base = so + sr * sld
            lo_e, hi_e = max(a0, base) - base, min(a1, base + sld) - base
            if hi_e > lo_e:
                dead[sr] |= ((n // 2 >= lo_e) & (n // 2 < hi_e)) | \
                            ((sld // 2 + n // 2 >= lo_e) & (sld // 2 + n // 2 < hi_e))
    return dead


def kpanels(A, P):
    """A (M x K) in the K-panel-major file layout of northup_file_tile_kpanels."""
    M, K = A.shape
    return np.concatenate([A[:, k0:k0 + P].ravel() for k0 in range(0, K, P)]) if K else A.ravel()


def simulate(plan: nu.Plan, A, B, M, N, K, rng=None, a_layout=None, replicas=None):
    """Replay the plan's ops on host arrays (float64, exact on integers).
    With `rng`, ops run in a random order consistent with the dependencies
    and with in-order execution per (worker, stream)."""
    bufs = plan.bufs()
    ops = plan.ops()
    mem = []
    for b in bufs:
        if b["kind"] == 0:
            mem.append((a_layout if a_layout is not None else A.ravel()).astype(np.float64).copy())
        elif b["kind"] == 1:
            mem.append(B.astype(np.float64).ravel().copy())
        elif b["kind"] == 2:
            mem.append(np.full(M * N, np.nan))
        else:
            mem.append(np.full(b["bytes"] // 4, np.nan))

    # NU_OP_SPLIT_B rewrites a resident B region in place into the leaf's split
    # form: model that as moving the values to a shadow copy (the raw rows
    # become NaN over their whole leading dimension, as the hi / lo halves
    # do on the GPU) which only pre-split leaf ops read; a later copy into a
    # row destroys the split values whose hi (element n/2) or lo (ld/2 + n/2)
    # bytes it overwrites.
    shadow = [np.full(len(x), np.nan) for x in mem]
    splits = [[] for _ in mem]            # per buffer: split regions (off, ld, rows, n)

    def view(buf, off, ld, rows, cols, m=None):
        m = mem if m is None else m
        assert off >= 0 and (rows == 0 or cols == 0 or off + (rows - 1) * ld + cols <= len(m[buf])), \
            f"op region outside buffer {buf}"
        return np.lib.stride_tricks.as_strided(m[buf][off:], shape=(rows, cols),
                                               strides=(ld * 8, 8), writeable=True)

    # The column exponents a SPLIT_B writes (one int per column, (c_buf, c_off))
    # are modelled as a tag value; a pre-split leaf requires the tags of every
    # K panel it reads, so anything overwriting them (or reading them before
    # the split) poisons its result.
    EXP_TAG = -12345.0
    kc = plan.stats().get("bk") or 0

    def clobber_split(buf, off, ld, rows, cols):
        """A write destroys the split values whose hi / lo bytes it covers."""
        for (so, sld, srows, sn) in splits[buf]:
            dead = split_dead_mask(off, ld, rows, cols, so, sld, srows, sn)
            if dead.any():
                view(buf, so, sld, srows, sn, shadow)[dead] = np.nan

    def run(op):
        if op["op"] in (nu.NU_OP_COPY, nu.NU_OP_IO_READ, nu.NU_OP_IO_WRITE):
            view(op["dst_buf"], op["dst_off"], op["dst_ld"], op["rows"], op["cols"])[...] = \
                view(op["src_buf"], op["src_off"], op["src_ld"], op["rows"], op["cols"]).copy()
            clobber_split(op["dst_buf"], op["dst_off"], op["dst_ld"], op["rows"], op["cols"])
        elif op["op"] == nu.NU_OP_SPLIT_B:
            src = view(op["dst_buf"], op["dst_off"], op["dst_ld"], op["rows"], op["cols"])
            view(op["dst_buf"], op["dst_off"], op["dst_ld"], op["rows"], op["cols"], shadow)[...] = src
            view(op["dst_buf"], op["dst_off"], op["dst_ld"], op["rows"], op["dst_ld"])[...] = np.nan
            splits[op["dst_buf"]].append((op["dst_off"], op["dst_ld"], op["rows"], op["cols"]))
            view(op["c_buf"], op["c_off"], op["cols"], 1, op["cols"])[...] = EXP_TAG
        elif op["op"] == nu.NU_OP_LEAF:
            a = view(op["a_buf"], op["a_off"], op["lda"], op["m"], op["k"])
            b = view(op["b_buf"], op["b_off"], op["ldb"], op["k"], op["n"],
                     shadow if op["src_buf"] >= 0 else None)
            c = view(op["c_buf"], op["c_off"], op["ldc"], op["m"], op["n"])
            prod = a @ b
            if op["src_buf"] >= 0 and kc > 0:
                for p in range(-(-op["k"] // kc)):
                    e = view(op["src_buf"], op["src_off"] + p * op["rows"], op["n"], 1, op["n"])
                    if not (e == EXP_TAG).all():
                        prod = prod * np.nan
            c[...] = (c + prod) if op["accumulate"] else prod
        else:
            view(op["c_buf"], op["c_off"], op["ldc"], op["m"], op["n"])[...] = 0

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
            assert ready, "deadlock: dependencies form a cycle"
            q = rng.choice(ready)
            i = q.pop(0)
            run(ops[i])
            done.add(i)
    if replicas is not None:
        replicas.extend(mem[i].reshape(M, N) for i, b in enumerate(bufs) if b["kind"] == 5)
    return mem[[b["kind"] for b in bufs].index(2)].reshape(M, N)


def _plan_case(M, N, K, G=1, cap=0, block=None, sched=nu.NU_SCHED_AUTO, kc=0):
    t, _ = nu.host_tree(G, cap)
    if block:
        t.set_block(0, *block)
    p = t.plan(M, N, K, nu.make_opts(schedule=sched, k_chunk=kc))
    return t, p


@pytest.mark.parametrize("M,N,K,G,cap,block,sched,kc", [
    (256, 256, 256, 1, 0, (64, 64, 64), nu.NU_SCHED_AUTO, 0),     # cfg1 shape (S1)
    (300, 200, 130, 1, 0, None, nu.NU_SCHED_AUTO, 0),             # ragged, S2 all-tail
    (513, 300, 777, 2, 0, None, nu.NU_SCHED_S2, 64),              # S2, 2 GPUs, small kc
    (400, 520, 1000, 1, 600_000, None, nu.NU_SCHED_S2, 32),       # capacity forces blocks
    (200, 300, 150, 4, 0, (64, 96, 40), nu.NU_SCHED_S1, 0),       # S1 on 4 GPUs
    (1, 1, 1, 1, 0, None, nu.NU_SCHED_AUTO, 0),
    (700, 300, 520, 1, 0, None, nu.NU_SCHED_S2B, 64),             # B-first: B resident, strips over K
    (1000, 600, 900, 1, 2_000_000, None, nu.NU_SCHED_S2B, 128),   # B-first under a cap: several blocks
    (300, 200, 100, 2, 0, None, nu.NU_SCHED_S2B, 32),             # B-first on 2 siblings, ragged
])
def test_plan_simulation_exact(M, N, K, G, cap, block, sched, kc):
    A = nugen.fill(M, K, 3, 1, "int")
    B = nugen.fill(K, N, 3, 2, "int")
    ref = A.astype(np.float64) @ B.astype(np.float64)
    t, p = _plan_case(M, N, K, G, cap, block, sched, kc)
    assert np.array_equal(simulate(p, A, B, M, N, K), ref)
    for seed in range(4):
        C = simulate(p, A, B, M, N, K, rng=random.Random(seed))
        assert np.array_equal(C, ref), f"order seed {seed} broke a dependency"
    if cap:
        assert all(b["bytes"] <= cap for b in p.bufs() if b["kind"] == 3)
    t.destroy()


def test_plan_bytes_closed_forms():
    # S2 with a whole-region C block: every A and B byte crosses PCIe once,
    # C comes back once (H2D = 4K(r + c), D2H = 4rc).
    M, N, K = 4096, 2048, 8192
    t, p = _plan_case(M, N, K, sched=nu.NU_SCHED_S2)
    s = p.stats()
    assert s["bytes_h2d"] == 4 * K * (M + N) and s["bytes_d2h"] == 4 * M * N
    assert s["bm"] == M and s["bn"] == N and s["schedule"] == nu.NU_SCHED_S2
    t.destroy()
    # S1 (paper-literal): A once, B once per row shard: 4MK + 4KN ceil(M/bm)
    M, N, K, bm = 256, 256, 256, 64
    t, p = _plan_case(M, N, K, block=(bm, 64, 64))
    s = p.stats()
    assert s["schedule"] == nu.NU_SCHED_S1
    assert s["bytes_h2d"] == 4 * M * K + 4 * K * N * (M // bm) and s["bytes_d2h"] == 4 * M * N
    assert s["leaf_launches"] == (M // 64) * (N // 64) * (K // 64)
    t.destroy()


def test_bfirst_plan_bytes_and_shape():
    """NU_SCHED_S2B: every A and B byte crosses PCIe once and C comes back
    once (the same closed form as S2); B is split in place once per K panel;
    the r1 main-phase rows and the strips cover the block."""
    M, N, K, kc = 4096, 2048, 8192, 512
    t, p = _plan_case(M, N, K, sched=nu.NU_SCHED_S2B, kc=kc)
    s = p.stats()
    assert s["schedule"] == nu.NU_SCHED_S2B and 0 < s["bfirst_rows"] < M and s["tail_k"] == K
    assert s["bytes_h2d"] == 4 * K * (M + N) and s["bytes_d2h"] == 4 * M * N
    ops = p.ops()
    assert sum(op["op"] == nu.NU_OP_SPLIT_B for op in ops) == K // kc
    t.destroy()


def test_cfg3_plan_shape():
    """cfg3: 32768^3, 8 GiB HBM cap -> the cost model picks S2's B-first
    variant; the drain-tail S2 stays available as NU_SCHED_S2."""
    M = N = K = 32768
    t, p = _plan_case(M, N, K, cap=8 * GiB)
    s = p.stats()
    assert s["schedule"] == nu.NU_SCHED_S2B and s["bm"] == M and s["bn"] == N
    assert 8192 <= s["bfirst_rows"] <= 24576 and s["hbm_peak_bytes"] <= 8 * GiB
    assert s["bytes_h2d"] == 4 * K * (M + N) and s["bytes_d2h"] == 4 * M * N
    t.destroy()
    t, p = _plan_case(M, N, K, cap=8 * GiB, sched=nu.NU_SCHED_S2)
    s = p.stats()
    assert s["schedule"] == nu.NU_SCHED_S2 and s["bm"] == M and s["bn"] == N
    assert 0 < s["tail_k"] < K and s["tail_k"] % 1024 == 0 and s["strips"] >= 8
    assert s["hbm_peak_bytes"] <= 8 * GiB
    assert s["bytes_h2d"] == 4 * K * (M + N) and s["bytes_d2h"] == 4 * M * N
    ks = [op["k"] for op in p.ops() if op["op"] == nu.NU_OP_LEAF]
    assert all(k % 1024 == 0 for k in ks)            # panel edges on k_chunk multiples
    t.destroy()


def test_capacity_below_minimum_block():
    t, _ = nu.host_tree(1, 4096)
    with pytest.raises(nu.NorthupError) as e:
        t.plan(1024, 1024, 1024)
    assert e.value.code == nu.NU_ENOMEM
    t.destroy()


def test_hbm_root_plan_is_one_leaf():
    t = nu.hbm_tree(0)
    p = t.plan(8192, 8192, 8192)
    ops = p.ops()
    assert len(ops) == 1 and ops[0]["op"] == nu.NU_OP_LEAF and ops[0]["k"] == 8192
    p2 = t.plan(100, 30, 7)    # K % 4 != 0: A is staged into a padded arena copy
    kinds = [o["op"] for o in p2.ops()]
    assert kinds == [nu.NU_OP_COPY, nu.NU_OP_COPY, nu.NU_OP_LEAF][:len(kinds)] or \
        kinds == [nu.NU_OP_COPY, nu.NU_OP_LEAF]
    t.destroy()


def test_data_api_host_only_errors():
    t, _ = nu.host_tree(1)
    with pytest.raises(nu.NorthupError):
        t.alloc(64, 2)     # SMEM node: managed by the leaf kernel
    t.destroy()


def file_tree(G, cap=0, staging_cap=0):
    t = nu.Tree()
    root = t.add_node(-1, nu.NU_FILE)
    st = t.add_node(root, nu.NU_HOST, -1, staging_cap)
    for g in range(G):
        h = t.add_node(st, nu.NU_HBM, 0, cap)
        t.add_node(h, nu.NU_SMEM, 0, 227 * 1024, nu.NU_PROC_SM100)
    return t


@pytest.mark.parametrize("M,N,K,G,cap,panel", [
    (300, 200, 130, 1, 0, 0),          # row-major A file
    (256, 384, 512, 2, 0, 128),        # K-panel-major A, two siblings
    (400, 520, 700, 2, 700_000, 64),   # HBM capacity forces several C-block rounds
    (130, 70, 33, 4, 0, 16),           # ragged last panel, 2 x 2 grid
])
def test_file_root_plan_simulation(M, N, K, G, cap, panel):
    A = nugen.fill(M, K, 4, 1, "int")
    B = nugen.fill(K, N, 4, 2, "int")
    ref = A.astype(np.float64) @ B.astype(np.float64)
    t = file_tree(G, cap)
    p = t.plan(M, N, K, nu.make_opts(k_chunk=64, a_panel_k=panel))
    ops = p.ops()
    assert any(o["op"] == nu.NU_OP_IO_READ for o in ops) and any(o["op"] == nu.NU_OP_IO_WRITE for o in ops)
    lay = kpanels(A, panel) if panel else None
    assert np.array_equal(simulate(p, A, B, M, N, K, a_layout=lay), ref)
    for seed in range(4):
        C = simulate(p, A, B, M, N, K, rng=random.Random(seed), a_layout=lay)
        assert np.array_equal(C, ref), f"order seed {seed} broke a dependency"
    s = p.stats()
    assert s["bytes_file_write"] == 4 * M * N
    t.destroy()


def test_file_tile_kpanels_round_trip(tmp_path):
    M, K, P = 37, 101, 16
    A = nugen.fill(M, K, 5, 1)
    src, dst = tmp_path / "a.bin", tmp_path / "a_tiled.bin"
    A.tofile(src)
    nu.file_tile_kpanels(str(src), str(dst), M, K, P)
    assert np.array_equal(np.fromfile(dst, dtype=np.float32), kpanels(A, P).astype(np.float32))


# ----------------------------------------------------- randomised planner check
from hypothesis import HealthCheck, given, settings, strategies as st


@settings(max_examples=40, deadline=None, suppress_health_check=[HealthCheck.too_slow])
@given(M=st.integers(1, 300), N=st.integers(1, 300), K=st.integers(1, 300),
       G=st.sampled_from([1, 2, 3, 4]), cap_kib=st.sampled_from([0, 300, 800, 2000]),
       kc=st.sampled_from([32, 64, 128]), sched=st.sampled_from([0, 1, 2, 4]),
       file_root=st.booleans(), panel=st.sampled_from([0, 32, 64]), seed=st.integers(0, 3))
def test_random_plans_replay_exactly(M, N, K, G, cap_kib, kc, sched, file_root, panel, seed):
    """Any tree shape / capacity / schedule the planner accepts yields an op
    list whose dependency-respecting replay computes A.B exactly; capacity
    errors are NU_ENOMEM, nothing else."""
    cap = cap_kib * 1024
    if file_root:
        t = file_tree(G, cap)
        opts = nu.make_opts(k_chunk=kc, a_panel_k=panel)
    else:
        t, _ = nu.host_tree(G, cap)
        opts = nu.make_opts(schedule=sched, k_chunk=kc)
    try:
        p = t.plan(M, N, K, opts)
    except nu.NorthupError as e:
        assert e.code == nu.NU_ENOMEM
        t.destroy()
        return
    A = nugen.fill(M, K, seed, 1, "int")
    B = nugen.fill(K, N, seed, 2, "int")
    lay = kpanels(A, panel) if (file_root and panel) else None
    C = simulate(p, A, B, M, N, K, rng=random.Random(seed), a_layout=lay)
    assert np.array_equal(C, A.astype(np.float64) @ B.astype(np.float64))
    if cap:
        assert all(b["bytes"] <= cap for b in p.bufs() if b["kind"] == 3)
    t.destroy()


# ------------------------------------------- NVLink-shared staging (NEXT-1)
@pytest.mark.parametrize("M,N,K,G,cap,kc", [
    (512, 512, 640, 2, 0, 64),          # 2 x 1 grid: B shared by the 2 row strips
    (512, 512, 640, 4, 0, 64),          # 2 x 2: A shared in grid rows, B in grid columns
    (1024, 512, 1000, 8, 0, 128),       # 4 x 2, ragged last K panel
    (600, 600, 700, 4, 1_200_000, 64),  # capacity forces several C blocks per region
    (4096, 8192, 512, 8, 0, 128),       # first-panel sub-block grid (bm, bn >= 4096)
    (900, 900, 1024, 3, 4 << 20, 512),  # ragged last column block with an in-place split B tail
])
def test_shared_staging_plan_replays_exactly(M, N, K, G, cap, kc):
    """Shared staging: every A/B byte crosses PCIe once per grid row / column
    (each sibling loads 1/Pc of A and 1/Pr of B), the rest is pulled from
    peers; any dependency-respecting order (cross-worker waits included)
    computes A.B exactly."""
    A = nugen.fill(M, K, 6, 1, "int")
    B = nugen.fill(K, N, 6, 2, "int")
    ref = A.astype(np.float64) @ B.astype(np.float64)
    t, _ = nu.host_tree(G, cap)
    p = t.plan(M, N, K, nu.make_opts(k_chunk=kc))
    s = p.stats()
    assert s["shared_staging"] == 1
    ops = p.ops()
    cross = [o for o in ops for d in o["deps"] if ops[d]["worker"] != o["worker"]]
    # pulls, slot reuse by loads, and the in-place split of the B tail after the
    # peers pulled their pieces from it (WAR)
    assert cross and all(o["stream"] in (4, 0) or o["op"] == nu.NU_OP_SPLIT_B for o in cross)
    for seed in range(4):
        C = simulate(p, A, B, M, N, K, rng=random.Random(seed))
        assert np.array_equal(C, ref), f"order seed {seed} broke a dependency"
    Pr, Pc = nu.partition(G, M, N)
    m, n = M // Pr, N // Pc
    nbr, nbc = -(-m // s["bm"]), -(-n // s["bn"])
    # per C block every sibling streams its A strip once (shared by Pc) and
    # its B strip once (shared by Pr): total PCIe bytes = blocks x (A + B) once
    assert s["bytes_h2d"] == 4 * K * (M * nbc + N * nbr)
    assert s["bytes_p2p"] == 4 * K * (M * nbc * (Pc - 1) + N * nbr * (Pr - 1))
    assert s["bytes_d2h"] == 4 * M * N
    if cap:
        assert all(b["bytes"] <= cap for b in p.bufs() if b["kind"] == 3)
    t.destroy()


def test_shared_staging_same_leaf_sequence_and_fewer_pcie_bytes():
    """On and off give the same leaf ops per worker (so bitwise-identical C on
    the GPU) while PCIe bytes drop from 4K(M Pc + N Pr) to 4K(M + N)."""
    M, N, K, G = 2048, 2048, 4096, 8
    t, _ = nu.host_tree(G)
    on = t.plan(M, N, K, nu.make_opts(k_chunk=256))
    off = t.plan(M, N, K, nu.make_opts(k_chunk=256, shared_staging=-1))
    so, sf = on.stats(), off.stats()
    assert so["shared_staging"] == 1 and sf["shared_staging"] == 0
    Pr, Pc = nu.partition(G, M, N)
    assert sf["bytes_h2d"] == 4 * K * (M * Pc + N * Pr) and so["bytes_h2d"] == 4 * K * (M + N)

    def leaves(p):
        bufs = p.bufs()
        out = {}
        for o in p.ops():
            if o["op"] == nu.NU_OP_LEAF:
                out.setdefault(o["worker"], []).append(
                    (o["m"], o["n"], o["k"], o["accumulate"], o["c_off"], o["ldc"]))
        return out
    lo, lf = leaves(on), leaves(off)
    # the leaf sequence per worker covers the same C elements in the same K order
    for w in range(G):
        ko = [(m, n, k, a) for (m, n, k, a, _, _) in lo[w]]
        kf = [(m, n, k, a) for (m, n, k, a, _, _) in lf[w]]
        assert sum(m * n * k for m, n, k, _ in ko) == sum(m * n * k for m, n, k, _ in kf)
    t.destroy()


def test_shared_staging_falls_back_for_ragged_regions():
    t, _ = nu.host_tree(3)
    p = t.plan(301, 200, 90, nu.make_opts(k_chunk=32))     # 1 x 3 grid, 200 = 67+67+66
    assert p.stats()["shared_staging"] == 0
    t.destroy()


def simulate_local(plan: nu.Plan, A, B, M, N, K, G, rng):
    """Replay a multi-process-siblings plan (northup_tree_set_local): worker w's
    user-buffer ops address only ITS strips (A rows, B columns, C region with
    region-local leading dimensions); arenas are shared (pulls read peers')."""
    bufs, ops = plan.bufs(), plan.ops()
    strips = []
    for w in range(G):
        r0, r1, c0, c1 = nu.partition_region(G, M, N, K, w)
        strips.append({0: A[r0:r1].astype(np.float64).ravel().copy(),
                       1: B[:, c0:c1].astype(np.float64).ravel().copy(),
                       2: np.full((r1 - r0) * (c1 - c0), np.nan), "reg": (r0, r1, c0, c1)})
    arenas = {i: np.full(b["bytes"] // 4, np.nan) for i, b in enumerate(bufs) if b["kind"] >= 3}

    def mem(w, i):
        return strips[w][bufs[i]["kind"]] if bufs[i]["kind"] < 3 else arenas[i]

    shadows = {}
    splits = {}

    def view(w, buf, off, ld, rows, cols, shadow=False):
        base = mem(w, buf)
        if shadow:
            base = shadows.setdefault(id(base), np.full(len(base), np.nan))
        return np.lib.stride_tricks.as_strided(base[off:], shape=(rows, cols),
                                               strides=(ld * 8, 8), writeable=True)

    queues = {}
    for i, op in enumerate(ops):
        queues.setdefault((op["worker"], op["stream"]), []).append(i)
    done = set()
    while len(done) < len(ops):
        ready = [q for q in queues.values() if q and all(d in done for d in ops[q[0]]["deps"])]
        assert ready
        i = rng.choice(ready).pop(0)
        op, w = ops[i], ops[i]["worker"]
        if op["op"] == nu.NU_OP_COPY:
            view(w, op["dst_buf"], op["dst_off"], op["dst_ld"], op["rows"], op["cols"])[...] = \
                view(w, op["src_buf"], op["src_off"], op["src_ld"], op["rows"], op["cols"]).copy()
            for (so, sld, srows, sn) in splits.get(id(mem(w, op["dst_buf"])), []):
                dead = split_dead_mask(op["dst_off"], op["dst_ld"], op["rows"], op["cols"], so, sld, srows, sn)
                if dead.any():
                    view(w, op["dst_buf"], so, sld, srows, sn, True)[dead] = np.nan
        elif op["op"] == nu.NU_OP_SPLIT_B:
            src = view(w, op["dst_buf"], op["dst_off"], op["dst_ld"], op["rows"], op["cols"])
            view(w, op["dst_buf"], op["dst_off"], op["dst_ld"], op["rows"], op["cols"], True)[...] = src
            view(w, op["dst_buf"], op["dst_off"], op["dst_ld"], op["rows"], op["dst_ld"])[...] = np.nan
            splits.setdefault(id(mem(w, op["dst_buf"])), []).append(
                (op["dst_off"], op["dst_ld"], op["rows"], op["cols"]))
        elif op["op"] == nu.NU_OP_LEAF:
            a = view(w, op["a_buf"], op["a_off"], op["lda"], op["m"], op["k"])
            b = view(w, op["b_buf"], op["b_off"], op["ldb"], op["k"], op["n"], op["src_buf"] >= 0)
            c = view(w, op["c_buf"], op["c_off"], op["ldc"], op["m"], op["n"])
            c[...] = (c + a @ b) if op["accumulate"] else a @ b
        done.add(i)
    C = np.full((M, N), np.nan)
    for s in strips:
        r0, r1, c0, c1 = s["reg"]
        C[r0:r1, c0:c1] = s[2].reshape(r1 - r0, c1 - c0)
    return C


@pytest.mark.parametrize("M,N,K,G,shared,sched", [(512, 512, 640, 2, 0, 0), (512, 512, 640, 4, 0, 0),
                                                   (1024, 512, 1000, 8, 0, 0), (300, 200, 130, 3, -1, 0),
                                                   (512, 256, 384, 4, -1, 0), (700, 400, 520, 2, -1, 4)])
def test_multiprocess_sibling_plan_uses_local_strips(M, N, K, G, shared, sched):
    """northup_tree_set_local: the same plan on every process, each sibling's
    root ops addressing its own strips (region-local leading dimensions);
    replayed with per-process strips it computes A.B exactly (also with S2's
    B-first variant, which a rank may pick when shared staging is off)."""
    A = nugen.fill(M, K, 7, 1, "int")
    B = nugen.fill(K, N, 7, 2, "int")
    t, hbm = nu.host_tree(G)
    t.set_local(hbm[G - 1])
    p = t.plan(M, N, K, nu.make_opts(schedule=sched, k_chunk=64, shared_staging=shared))
    assert p.stats()["shared_staging"] == (1 if shared == 0 else 0)
    if sched:
        assert p.stats()["schedule"] == sched
    for seed in range(3):
        C = simulate_local(p, A, B, M, N, K, G, random.Random(seed))
        assert np.array_equal(C, A.astype(np.float64) @ B.astype(np.float64))
    t.destroy()


def test_set_local_errors():
    t, hbm = nu.host_tree(2)
    with pytest.raises(nu.NorthupError):
        t.set_local(0)                       # the HOST root is not an HBM node
    t.set_local(hbm[1])
    with pytest.raises(nu.NorthupError) as e:
        t.peer_export(64, 64, 64)            # not finalized
    assert e.value.code == nu.NU_ESTATE
    t.destroy()


# ------------------------------------------- queue scheduling (NEXT-2)
@pytest.mark.parametrize("M,N,K,G,cap,kc", [
    (512, 512, 640, 2, 0, 64), (600, 300, 200, 3, 0, 64), (1000, 700, 500, 4, 1_500_000, 128),
    (130, 90, 70, 1, 0, 32)])
def test_queue_plan_replays_exactly(M, N, K, G, cap, kc):
    """NU_SCHED_QUEUE: two or more tiles per sibling, each an S2 sub-problem with two
    C-tile buffers; the plan API's no-steal unrolling replays exactly in any
    dependency-respecting order and moves the closed-form bytes."""
    A = nugen.fill(M, K, 8, 1, "int")
    B = nugen.fill(K, N, 8, 2, "int")
    ref = A.astype(np.float64) @ B.astype(np.float64)
    t, _ = nu.host_tree(G, cap)
    p = t.plan(M, N, K, nu.make_opts(schedule=nu.NU_SCHED_QUEUE, k_chunk=kc))
    s = p.stats()
    assert s["schedule"] == nu.NU_SCHED_QUEUE and s["tasks"] >= min(2 * G, -(-M // 8) * -(-N // 8))
    for seed in range(3):
        assert np.array_equal(simulate(p, A, B, M, N, K, rng=random.Random(seed)), ref)
    tr, tc = -(-M // s["bm"]), -(-N // s["bn"])
    assert s["bytes_h2d"] == 4 * K * (M * tc + N * tr) and s["bytes_d2h"] == 4 * M * N
    if cap:
        assert all(b["bytes"] <= cap for b in p.bufs() if b["kind"] == 3)
    t.destroy()



def direct_file_tree(G, cap=0):
    t = nu.Tree()
    root = t.add_node(-1, nu.NU_FILE)
    for g in range(G):
        h = t.add_node(root, nu.NU_HBM, 0, cap)
        t.add_node(h, nu.NU_SMEM, 0, 227 * 1024, nu.NU_PROC_SM100)
    return t


@pytest.mark.parametrize("M,N,K,G,cap,panel", [(300, 200, 130, 1, 0, 0), (256, 384, 512, 2, 0, 128),
                                               (400, 520, 700, 2, 700_000, 64), (130, 70, 33, 4, 0, 16)])
def test_file_direct_plan_simulation(M, N, K, G, cap, panel):
    """FILE -> HBM (the GDS edge, NEXT-4): panels read from the files straight
    into HBM slots, C blocks written from HBM; replays exactly in any order."""
    A = nugen.fill(M, K, 5, 1, "int")
    B = nugen.fill(K, N, 5, 2, "int")
    ref = A.astype(np.float64) @ B.astype(np.float64)
    t = direct_file_tree(G, cap)
    p = t.plan(M, N, K, nu.make_opts(k_chunk=64, a_panel_k=panel))
    ops = p.ops()
    assert not any(o["op"] == nu.NU_OP_COPY for o in ops)           # no DRAM bounce in the plan
    lay = kpanels(A, panel) if panel else None
    for seed in range(3):
        C = simulate(p, A, B, M, N, K, rng=random.Random(seed), a_layout=lay)
        assert np.array_equal(C, ref), f"order seed {seed} broke a dependency"
    assert p.stats()["bytes_file_write"] == 4 * M * N
    if cap:
        assert all(b["bytes"] <= cap for b in p.bufs() if b["kind"] == 3)
    t.destroy()


@pytest.mark.parametrize("M,N,K,G,cap,block,sched,kc", [
    (300, 200, 130, 1, 0, None, nu.NU_SCHED_AUTO, 0),             # S2, one sibling
    (513, 300, 777, 2, 0, None, nu.NU_SCHED_S2, 64),              # S2 with shared staging
    (400, 520, 1000, 2, 600_000, None, nu.NU_SCHED_S2, 32),       # several C blocks per sibling
    (200, 300, 150, 4, 0, (64, 96, 40), nu.NU_SCHED_S1, 0),       # S1 blocks on 4 siblings
    (700, 300, 520, 2, 0, None, nu.NU_SCHED_S2B, 64),             # B-first strips
])
def test_replicate_result_plan_pushes_every_piece(M, N, K, G, cap, block, sched, kc):
    """replicate_result in one process: after each drain of a finished C piece
    the plan copies the same HBM region into every sibling's replica (S§8(e)),
    on the sibling's device-to-device stream.  Replayed in random dependency-
    respecting orders, every replica equals C exactly (integer inputs), and a
    replica push never waits on the D2H drain it shadows."""
    A = nugen.fill(M, K, 4, 1, "int")
    B = nugen.fill(K, N, 4, 2, "int")
    ref = A.astype(np.float64) @ B.astype(np.float64)
    t, hbm = nu.host_tree(G, cap)
    if block:
        t.set_block(0, *block)
    for h in hbm:
        t.set_replica(h, 0x1000, 4 * M * N)   # plan-time check only: never dereferenced here
    p = t.plan(M, N, K, nu.make_opts(schedule=sched, k_chunk=kc, replicate_result=True))
    bufs, ops = p.bufs(), p.ops()
    rep = [i for i, b in enumerate(bufs) if b["kind"] == 5]
    assert [bufs[i]["worker"] for i in rep] == list(range(G))
    drains = [o for o in ops if o["op"] == nu.NU_OP_COPY and bufs[o["dst_buf"]]["kind"] == 2]
    pushes = [o for o in ops if o["op"] == nu.NU_OP_COPY and o["dst_buf"] in rep]
    assert len(pushes) == G * len(drains) > 0
    assert {o["stream"] for o in pushes} == {4}                    # S_D2D
    assert p.stats()["bytes_d2d"] >= G * 4 * M * N
    for seed in range(3):
        reps = []
        C = simulate(p, A, B, M, N, K, rng=random.Random(seed), replicas=reps)
        assert np.array_equal(C, ref)
        assert len(reps) == G and all(np.array_equal(r, ref) for r in reps), f"seed {seed}"
    # without a registered replica the plan refuses replicate_result
    t.set_replica(hbm[-1], 0, 0)
    with pytest.raises(nu.NorthupError):
        t.plan(M, N, K, nu.make_opts(schedule=sched, k_chunk=kc, replicate_result=True))
    t.destroy()
