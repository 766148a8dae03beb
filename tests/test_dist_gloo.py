"""Multi-process C-subtree partition (S§8(e)) with world_size 2 and 4 over
gloo on CPU: every rank owns a disjoint region; the regions tile C exactly;
the gather assembles the full C.  The per-rank GEMM here is the CPU plan
simulator replaying northup's own plan for the rank's region (no GPU)."""
import os
import random

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import nugen


def _rank_main(rank, world, port, M, N, K, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import paper_conf_ipps_chey19_b200 as nu
        from paper_conf_ipps_chey19_b200.dist import gather_regions, my_region
        from test_capi_host import simulate
        r0, r1, c0, c1 = my_region(M, N, K, rank, world)
        # inputs of the region only, regenerated from global coordinates
        A = nugen.fill(r1 - r0, K, 7, 1, "int", i0=r0, ncols=K)
        B = nugen.fill(K, c1 - c0, 7, 2, "int", j0=c0, ncols=N)
        t, _ = nu.host_tree(1)
        p = t.plan(r1 - r0, c1 - c0, K, nu.make_opts(k_chunk=64))
        Creg = simulate(p, A, B, r1 - r0, c1 - c0, K, rng=random.Random(rank))
        t.destroy()
        full = gather_regions(torch.from_numpy(Creg), M, N, K, rank, world)
        q.put((rank, full.numpy()))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,M,N,K", [(2, 130, 90, 70), (4, 96, 200, 33)])
def test_partitioned_gemm_and_gather_gloo(world, M, N, K):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + random.randint(0, 2000)
    procs = [ctx.Process(target=_rank_main, args=(r, world, port, M, N, K, q)) for r in range(world)]
    for p in procs:
        p.start()
    outs = dict(q.get(timeout=300) for _ in range(world))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    A = nugen.fill(M, K, 7, 1, "int")
    B = nugen.fill(K, N, 7, 2, "int")
    ref = A.astype(np.float64) @ B.astype(np.float64)
    for r in range(world):
        assert np.array_equal(outs[r], ref)


def _plan_rank(rank, world, port, M, N, K, q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import hashlib

        import paper_conf_ipps_chey19_b200 as nu
        t, hbm = nu.host_tree(world)
        t.set_local(hbm[rank])          # multi-process siblings: this rank's node
        p = t.plan(M, N, K, nu.make_opts(k_chunk=64))
        ops = p.ops()
        h = hashlib.sha256(repr([sorted(o.items()) for o in ops]).encode()).hexdigest()
        t.destroy()
        hs = [None] * world
        dist.all_gather_object(hs, h)
        q.put((rank, hs, p.stats()["shared_staging"]))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 4])
def test_multiprocess_siblings_plan_identically_gloo(world):
    """The cross-process protocol of multi-process siblings (peer flag words
    indexed by op) needs every rank to build the same op list whatever its
    local node: checked by all-gathering a hash of each rank's plan."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = 29500 + random.randint(2001, 4000)
    procs = [ctx.Process(target=_plan_rank, args=(r, world, port, 512, 512, 640, q)) for r in range(world)]
    for p in procs:
        p.start()
    outs = dict((r, (hs, sh)) for r, hs, sh in (q.get(timeout=300) for _ in range(world)))
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    hs0 = outs[0][0]
    assert len(set(hs0)) == 1 and all(outs[r][0] == hs0 for r in range(world))
    assert all(outs[r][1] == 1 for r in range(world))
