"""End-to-end parity of northup_gemm through the C ABI: HOST root -> HBM ->
SMEM/TMEM leaf (and the in-HBM single-node tree), against the fp64 oracle on
the same seeded inputs."""
import ctypes

import numpy as np
import pytest
import torch

import nugen
import oracle
import paper_conf_ipps_chey19_b200 as nu

pytestmark = pytest.mark.gpu
TOL = 1e-5
GiB = 1 << 30


def host_view(buf, rows, cols):
    n = rows * cols
    if n == 0:
        return np.zeros((rows, cols), np.float32)
    arr = (ctypes.c_float * n).from_address(buf.ptr)
    return np.ctypeslib.as_array(arr).reshape(rows, cols)


class HostProblem:
    """A, B, C allocated at the HOST root through Table I's alloc()."""

    def __init__(self, tree, M, N, K, seed, kind="uniform"):
        self.M, self.N, self.K = M, N, K
        self.A = tree.alloc(4 * M * K, 0)
        self.B = tree.alloc(4 * K * N, 0)
        self.C = tree.alloc(4 * M * N, 0)
        self.a = host_view(self.A, M, K)
        self.b = host_view(self.B, K, N)
        self.c = host_view(self.C, M, N)
        nugen.fill(M, K, seed, nugen.MAT_A, kind, out=self.a)
        nugen.fill(K, N, seed, nugen.MAT_B, kind, out=self.b)
        if M * N:
            self.c[...] = np.nan


def run_host(M, N, K, G=1, cap=0, block=None, kind="uniform", seed=1, **opt):
    t, _ = nu.host_tree(G, cap, devices=[0] * G)     # G "virtual siblings" on GPU 0 (T5)
    if block:
        t.set_block(0, *block)
    t.finalize()
    p = HostProblem(t, M, N, K, seed, kind)
    st = t.gemm(p.A, p.B, p.C, M, N, K, nu.make_opts(**opt))
    C = p.c.copy()
    a, b = p.a.copy(), p.b.copy()
    t.destroy()
    return C, a, b, st


def check(C, a, b, kind):
    ref = oracle.gemm(a, b)
    if kind == "int":
        assert np.array_equal(C.astype(np.float64), ref)
    else:
        e, where = oracle.normwise_err(C, ref, oracle.row_norms(a), oracle.col_norms(b))
        assert e <= TOL, (e, where)


def test_cfg1_two_level_tree_64_blocks():
    """BASELINE.json configs[0]: 256^3, host DRAM -> 1 GPU leaf, 64 x 64 blocks."""
    for kind in ("uniform", "int"):
        C, a, b, st = run_host(256, 256, 256, block=(64, 64, 64), kind=kind)
        check(C, a, b, kind)
        assert st["schedule"] == nu.NU_SCHED_S1 and st["leaf_launches"] == 64


@pytest.mark.parametrize("M,N,K,G,cap,sched,kc", [
    (300, 200, 130, 1, 0, 0, 0),
    (1, 1, 1, 1, 0, 0, 0),
    (513, 777, 2100, 1, 0, nu.NU_SCHED_S2, 256),
    (1000, 1200, 3000, 1, 6_000_000, nu.NU_SCHED_S2, 512),   # capacity -> several C blocks
    (640, 900, 1500, 2, 0, 0, 0),                            # 2 siblings, one device
    (500, 700, 333, 4, 0, nu.NU_SCHED_S1, 0),
    (2048, 2048, 12288, 1, 0, nu.NU_SCHED_S2, 1024),         # main phase + drain tail
    (2048, 1536, 6144, 1, 0, nu.NU_SCHED_S2B, 1024),         # B-first: B resident, strips over K
    (1000, 1200, 3000, 1, 9_000_000, nu.NU_SCHED_S2B, 512),  # B-first, capacity -> several blocks
    (700, 520, 900, 2, 0, nu.NU_SCHED_S2B, 128),             # B-first, 2 siblings, ragged
])
@pytest.mark.parametrize("kind", ["uniform", "int"])
def test_host_root_gemm(M, N, K, G, cap, sched, kc, kind):
    C, a, b, st = run_host(M, N, K, G=G, cap=cap, schedule=sched, k_chunk=kc, kind=kind)
    check(C, a, b, kind)
    assert st["num_gpus"] == G


@pytest.mark.parametrize("M,N,K,G,cap,sched,kc,block", [
    (1000, 1200, 3000, 1, 6_000_000, nu.NU_SCHED_S2, 256, None),     # several C blocks, slots reused
    (2048, 1536, 6144, 1, 0, nu.NU_SCHED_S2B, 512, None),            # B-first strips and C-strip slots
    (640, 900, 1500, 2, 0, nu.NU_SCHED_S2, 256, None),               # shared staging between siblings
    (512, 512, 512, 1, 0, nu.NU_SCHED_S1, 0, (128, 128, 128)),       # S1: row shard kept, blocks drained
])
def test_slot_reuse_under_slow_compute(monkeypatch, M, N, K, G, cap, sched, kc, block):
    """SURVEY T2's race test: sibling 0's compute stream is held for 50x each
    leaf's nominal time (NORTHUP_DEBUG_SLOW_SIBLING), so the copy streams run far
    ahead of the leaves and every slot reuse, C-strip drain and shared-staging
    pull must wait on its recorded dependency; integer inputs stay exact."""
    monkeypatch.setenv("NORTHUP_DEBUG_SLOW_SIBLING", "0,5000")
    C, a, b, st = run_host(M, N, K, G=G, cap=cap, block=block, schedule=sched, k_chunk=kc, kind="int", seed=7)
    check(C, a, b, "int")
    assert st["copies"] > 3


@pytest.mark.parametrize("M,N,K", [(1, 4097, 300), (4097, 1, 300), (257, 3, 1), (3, 5, 70000), (33, 2049, 7)])
def test_host_root_skinny_and_ragged(M, N, K):
    """Degenerate shapes through the HOST -> HBM tree (vectors, K = 1, a long K
    against a tiny C, ragged edges in every dimension): exact on integer inputs,
    within the bound on uniform ones."""
    for kind in ("int", "uniform"):
        C, a, b, st = run_host(M, N, K, kind=kind)
        check(C, a, b, kind)


def test_zero_k_and_empty():
    C, a, b, st = run_host(7, 9, 0)
    assert (C == 0).all()
    run_host(0, 5, 5)
    run_host(5, 0, 5)


def test_in_hbm_tree_and_cross_tier_bitwise():
    """CS4: the single-node HBM tree runs the same leaf; with K-panel edges on
    k_chunk multiples the out-of-core result is bitwise identical (§8(c) (4))."""
    M, N, K = 1536, 1024, 6144
    C_ooc, a, b, st = run_host(M, N, K, schedule=nu.NU_SCHED_S2, k_chunk=1024)
    assert st["tail_k"] > 0 and st["leaf_launches"] > 1
    dev = torch.device("cuda:0")
    Ad = torch.from_numpy(a).to(dev)
    Bd = torch.from_numpy(b).to(dev)
    Cd = torch.full((M, N), float("nan"), device=dev)
    t = nu.hbm_tree(0)
    t.finalize()
    bA = t.wrap_device(0, Ad.data_ptr(), Ad.numel() * 4)
    bB = t.wrap_device(0, Bd.data_ptr(), Bd.numel() * 4)
    bC = t.wrap_device(0, Cd.data_ptr(), Cd.numel() * 4)
    t.gemm(bA, bB, bC, M, N, K, nu.make_opts(k_chunk=1024))
    torch.cuda.synchronize()
    C_hbm = Cd.cpu().numpy()
    t.destroy()
    check(C_hbm, a, b, "uniform")
    assert np.array_equal(C_hbm, C_ooc)


def test_bfirst_bitwise_equals_drain_tail_and_in_hbm():
    """S2's B-first variant runs the same K-panel sequence per C element as
    the drain-tail S2 and the in-HBM tree (phase-1 rows panel by panel, strip
    rows as one leaf call over all panels of the pre-split B), so all three
    are bitwise equal (reading R20)."""
    M, N, K, kc = 4096, 3072, 8192, 1024
    C_b, a, b, st_b = run_host(M, N, K, schedule=nu.NU_SCHED_S2B, k_chunk=kc)
    assert st_b["schedule"] == nu.NU_SCHED_S2B and 0 < st_b["bfirst_rows"] < M
    C_s, _, _, st_s = run_host(M, N, K, schedule=nu.NU_SCHED_S2, k_chunk=kc)
    assert st_s["schedule"] == nu.NU_SCHED_S2
    check(C_b, a, b, "uniform")
    assert np.array_equal(C_b, C_s)
    dev = torch.device("cuda:0")
    Ad, Bd = torch.from_numpy(a).to(dev), torch.from_numpy(b).to(dev)
    Cd = torch.full((M, N), float("nan"), device=dev)
    t = nu.hbm_tree(0)
    t.finalize()
    t.gemm(t.wrap_device(0, Ad.data_ptr(), Ad.numel() * 4), t.wrap_device(0, Bd.data_ptr(), Bd.numel() * 4),
           t.wrap_device(0, Cd.data_ptr(), Cd.numel() * 4), M, N, K, nu.make_opts(k_chunk=kc))
    torch.cuda.synchronize()
    assert np.array_equal(Cd.cpu().numpy(), C_b)
    t.destroy()


def test_in_hbm_unaligned_operands_staged():
    """K % 4 != 0: the HBM root stages A into a padded arena (R16)."""
    M, N, K = 130, 66, 37
    a = nugen.fill(M, K, 5, 1, "int")
    b = nugen.fill(K, N, 5, 2, "int")
    dev = torch.device("cuda:0")
    Ad, Bd = torch.from_numpy(a).to(dev), torch.from_numpy(b).to(dev)
    Cd = torch.zeros((M, N), device=dev)
    t = nu.hbm_tree(0)
    t.finalize()
    st = t.gemm(t.wrap_device(0, Ad.data_ptr(), Ad.numel() * 4),
                t.wrap_device(0, Bd.data_ptr(), Bd.numel() * 4),
                t.wrap_device(0, Cd.data_ptr(), Cd.numel() * 4), M, N, K)
    assert st["bytes_d2d"] > 0
    assert np.array_equal(Cd.cpu().numpy().astype(np.float64), oracle.gemm(a, b))
    t.destroy()


def test_cross_g_bitwise():
    """Same K-panel sequence on G = 1 / 2 / 4 siblings gives identical C."""
    M, N, K = 1024, 768, 4096
    outs = [run_host(M, N, K, G=G, schedule=nu.NU_SCHED_S2, k_chunk=1024)[0] for G in (1, 2, 4)]
    assert np.array_equal(outs[0], outs[1]) and np.array_equal(outs[0], outs[2])


def test_data_api_round_trip():
    """Table I: alloc at HOST and HBM, move_data down and up, byte exact."""
    t, hbm = nu.host_tree(1)
    t.finalize()
    h = t.alloc(1 << 20, 0)
    d = t.alloc(1 << 20, hbm[0])
    back = t.alloc(1 << 20, 0)
    x = host_view(h, 256, 1024)
    x[...] = nugen.fill(256, 1024, 9, 1)
    t.move_data_down(d, h, 1 << 20, 0, 0)
    t.move_data_up(back, d, 1 << 20, 0)
    assert np.array_equal(host_view(back, 256, 1024), x)
    assert t.node_info(hbm[0])["used"] >= 1 << 20
    t.destroy()


def test_hbm_capacity_enforced():
    t, hbm = nu.host_tree(1, 1 << 20)
    t.finalize()
    with pytest.raises(nu.NorthupError) as e:
        t.alloc(2 << 20, hbm[0])
    assert e.value.code == nu.NU_ENOMEM
    t.destroy()


@pytest.mark.parametrize("G,sched,block", [(1, nu.NU_SCHED_AUTO, None), (2, nu.NU_SCHED_AUTO, None),
                                            (4, nu.NU_SCHED_AUTO, None), (2, nu.NU_SCHED_S1, (64, 96, 128)),
                                            (2, nu.NU_SCHED_S2B, None), (1, nu.NU_SCHED_S2B, None),
                                            (2, nu.NU_SCHED_QUEUE, None)])
def test_replicate_result(G, sched, block):
    """S§8(e) replicate_result: every sibling's HBM replica holds the whole C
    (G = 1; G > 1 as virtual siblings on one device).  The plan pushes each
    drained C piece into every replica on the device-to-device stream while
    the rest of the GEMM runs (no gather after the join)."""
    M, N, K = 700, 520, 900
    t, hbm = nu.host_tree(G, devices=[0] * G)
    if block:
        t.set_block(0, *block)
    t.finalize()
    p = HostProblem(t, M, N, K, 3, "int")
    reps = [torch.full((M, N), float("nan"), device="cuda:0") for _ in range(G)]
    for h, r in zip(hbm, reps):
        t.set_replica(h, r.data_ptr(), r.numel() * 4)
    st = t.gemm(p.A, p.B, p.C, M, N, K, nu.make_opts(schedule=sched, replicate_result=True))
    ref = oracle.gemm(p.a, p.b)
    assert np.array_equal(p.c.astype(np.float64), ref)
    for r in reps:
        assert np.array_equal(r.cpu().numpy().astype(np.float64), ref)
    if sched != nu.NU_SCHED_QUEUE:                 # the queue schedule gathers after the join
        assert st["bytes_d2d"] >= G * 4 * M * N    # the plan's pushes carried every replica
    t.destroy()


def test_replicate_result_graph_replay():
    """opts.graph with replicate_result: the captured op lists include the
    replica pushes, so a replayed call refreshes every replica."""
    M, N, K, G = 640, 384, 512, 2
    t, hbm = nu.host_tree(G, devices=[0] * G)
    t.finalize()
    p = HostProblem(t, M, N, K, 9, "int")
    reps = [torch.full((M, N), float("nan"), device="cuda:0") for _ in range(G)]
    for h, r in zip(hbm, reps):
        t.set_replica(h, r.data_ptr(), r.numel() * 4)
    o = nu.make_opts(replicate_result=True, graph=True, shared_staging=-1)
    ref = oracle.gemm(p.a, p.b)
    st1 = t.gemm(p.A, p.B, p.C, M, N, K, o)
    for r in reps:
        r.fill_(float("nan"))
    st2 = t.gemm(p.A, p.B, p.C, M, N, K, o)
    assert st2["graph_replayed"] == 1
    assert np.array_equal(p.c.astype(np.float64), ref)
    for r in reps:
        assert np.array_equal(r.cpu().numpy().astype(np.float64), ref)
    t.destroy()


def test_replicate_result_in_hbm_root_gathers():
    """A single-node HBM tree has no drains to piggy-back on: replicate_result
    copies the finished C into the replica after the join."""
    M, N, K = 300, 260, 200
    a = nugen.fill(M, K, 5, 1, "int")
    b = nugen.fill(K, N, 5, 2, "int")
    t = nu.hbm_tree(0)
    t.finalize()
    dev = torch.device("cuda", 0)
    A, B = torch.from_numpy(a).to(dev), torch.from_numpy(b).to(dev)
    C = torch.full((M, N), float("nan"), device=dev)
    rep = torch.full((M, N), float("nan"), device=dev)
    t.set_replica(0, rep.data_ptr(), rep.numel() * 4)
    bA, bB, bC = (t.wrap_device(0, x.data_ptr(), x.numel() * 4) for x in (A, B, C))
    t.gemm(bA, bB, bC, M, N, K, nu.make_opts(replicate_result=True))
    ref = oracle.gemm(a, b)
    assert np.array_equal(C.cpu().numpy().astype(np.float64), ref)
    assert np.array_equal(rep.cpu().numpy().astype(np.float64), ref)
    t.destroy()


@pytest.mark.parametrize("G,block,sched", [(1, (64, 64, 64), 0), (2, None, 0), (1, None, nu.NU_SCHED_S2B)])
def test_graph_capture_and_replay(G, block, sched):
    """opts.graph: the first call captures each GPU's op list into a CUDA graph,
    identical later calls replay it; results are bitwise the same."""
    M, N, K = 512, 384, 640
    t, _ = nu.host_tree(G, devices=[0] * G)
    if block:
        t.set_block(0, *block)
    t.finalize()
    p = HostProblem(t, M, N, K, 8, "int")
    o = nu.make_opts(graph=True, shared_staging=-1, schedule=sched, k_chunk=128 if sched else 0)
    st1 = t.gemm(p.A, p.B, p.C, M, N, K, o)
    c1 = p.c.copy()
    p.c[...] = np.nan
    st2 = t.gemm(p.A, p.B, p.C, M, N, K, o)
    assert st1["graph_replayed"] == 0 and st2["graph_replayed"] == 1
    assert np.array_equal(c1, p.c)
    assert np.array_equal(p.c.astype(np.float64), oracle.gemm(p.a, p.b))
    t.destroy()


@pytest.mark.parametrize("G,M,N,K,cap,kind", [
    (2, 1024, 768, 4096, 0, "uniform"),
    (4, 1024, 1024, 3000, 0, "int"),
    (8, 2048, 1024, 2048, 0, "uniform"),
    (4, 1536, 1536, 2560, 6 << 20, "int"),      # capacity: several C blocks per sibling
])
def test_shared_staging_virtual_siblings(G, M, N, K, cap, kind):
    """NEXT-1 shared staging on G virtual siblings of GPU 0: each sibling loads
    its piece of every panel over PCIe and pulls the rest from its peers'
    arenas (cross-worker event waits); C is bitwise identical to the unshared
    plan and matches the oracle."""
    kc = 512
    C1, a, b, s1 = run_host(M, N, K, G=G, cap=cap, kind=kind, seed=4, k_chunk=kc, collect_timing=True)
    C0, _, _, s0 = run_host(M, N, K, G=G, cap=cap, kind=kind, seed=4, k_chunk=kc, shared_staging=-1)
    assert s1["shared_staging"] == 1 and s0["shared_staging"] == 0
    assert s1["bytes_p2p"] > 0 and s1["bytes_h2d"] < s0["bytes_h2d"] and s1["t_p2p_ms"] > 0
    assert np.array_equal(C1, C0)
    check(C1, a, b, kind)


@pytest.mark.parametrize("G,M,N,K,cap,kind", [(2, 1024, 768, 2048, 0, "int"), (4, 1500, 1300, 1100, 0, "uniform"),
                                               (3, 900, 900, 1024, 4 << 20, "uniform")])
def test_queue_schedule_matches_static_and_oracle(G, M, N, K, cap, kind):
    """NEXT-2: tiles popped from per-sibling queues at run time give the
    oracle's C, bitwise equal to the static S2 plan (same K-chunk sequence
    per element)."""
    Cq, a, b, sq = run_host(M, N, K, G=G, cap=cap, kind=kind, seed=6, k_chunk=512,
                            schedule=nu.NU_SCHED_QUEUE)
    Cs, _, _, _ = run_host(M, N, K, G=G, cap=cap, kind=kind, seed=6, k_chunk=512, schedule=nu.NU_SCHED_S2)
    assert sq["schedule"] == nu.NU_SCHED_QUEUE and sq["tasks"] >= 2 * G
    check(Cq, a, b, kind)
    assert np.array_equal(Cq, Cs)


def test_queue_schedule_steals_from_a_slow_sibling(monkeypatch):
    """A sibling that is slow to pop (test hook emulating an asymmetric tree,
    Fig. 2) loses tiles to the fast one: steals happen and C is still exact."""
    # sibling 1 holds its compute stream 500x the nominal leaf time (2mnk at
    # 300 TF/s, ~1 ms here) before each leaf: the two virtual siblings share one
    # GPU and one PCIe link, so the delay must exceed a tile's copies to show
    monkeypatch.setenv("NORTHUP_DEBUG_SLOW_SIBLING", "1,50000")
    M, N, K = 2048, 2048, 1024
    C, a, b, st = run_host(M, N, K, G=2, kind="int", seed=2, k_chunk=512, schedule=nu.NU_SCHED_QUEUE,
                           queue_tiles=8)
    assert st["tasks_stolen"] > 0
    check(C, a, b, "int")


def test_finalize_measures_links():
    """finalize calibrates the planner's PCIe term with every local link busy
    (S§8(d)), records P2P reachability (shared staging needs it) and binds
    workers to their GPU's NUMA node when the host reports one."""
    t, _ = nu.host_tree(2, 1 << 30, devices=[0, 0])     # two virtual siblings on one GPU
    t.finalize()
    li = t.link_info()
    assert 10 < li["pcie_gbs"] < 80 and li["p2p_ok"]
    t.destroy()
    th = nu.hbm_tree(0)
    th.finalize()
    assert th.link_info()["pcie_gbs"] == 0.0            # no host edge, nothing measured
    th.destroy()
