"""Multi-process siblings (northup_tree_set_local + CUDA IPC peer export/import,
S§8(e) process model) with NVLink-shared staging (NEXT-1): G processes on the
one GPU of this pool, each running one HBM sibling; pulls read the peers'
arenas through IPC, cross-process dependencies are device-side flag waits.
The assembled C matches the oracle and is bitwise identical to the unshared
run and across repeated calls (generations)."""
import os
import subprocess
import sys

import numpy as np
import pytest

import nugen
import oracle
import paper_conf_ipps_chey19_b200 as nu

pytestmark = pytest.mark.gpu
HERE = os.path.dirname(os.path.abspath(__file__))


def spawn(tmp, G, M, N, K, kc, shared, kind, reps, env=None):
    d = tmp / f"rdv_{G}_{shared}_{kind}"
    d.mkdir()
    procs = [subprocess.Popen([sys.executable, os.path.join(HERE, "peer_sibling.py"), str(d), str(r),
                               str(G), str(M), str(N), str(K), str(kc), str(shared), kind, str(reps)],
                              stdout=subprocess.PIPE, stderr=subprocess.STDOUT, env=env)
             for r in range(G)]
    return d, procs


def run_siblings(tmp, G, M, N, K, kc, shared, kind, reps=2):
    d, procs = spawn(tmp, G, M, N, K, kc, shared, kind, reps)
    outs = []
    for p in procs:
        try:
            out, _ = p.communicate(timeout=300)
        except subprocess.TimeoutExpired:
            for q in procs:
                q.kill()
            raise
        outs.append(out.decode(errors="replace"))
    assert all(p.returncode == 0 for p in procs), "\n".join(outs)
    C = np.full((reps, M, N), np.nan, np.float32)
    stats = []
    for r in range(G):
        r0, r1, c0, c1 = nu.partition_region(G, M, N, K, r)
        C[:, r0:r1, c0:c1] = np.load(d / f"c{r}.npy")
        stats.append(list(map(int, open(d / f"st{r}.txt").read().split())))
    return C, stats


@pytest.mark.parametrize("G,M,N,K,kind", [(2, 1024, 768, 3072, "int"), (4, 1024, 1024, 2048, "uniform")])
def test_multiprocess_shared_staging(tmp_path, G, M, N, K, kind):
    kc = 512
    Cs, st = run_siblings(tmp_path, G, M, N, K, kc, 0, kind)
    Cu, su = run_siblings(tmp_path, G, M, N, K, kc, -1, kind)
    assert all(s[0] == 1 and s[1] > 0 for s in st) and all(s[0] == 0 for s in su)
    assert np.array_equal(Cs[0], Cs[1])            # generation 2 == generation 1
    assert np.array_equal(Cs[0], Cu[0])            # shared == unshared, bitwise
    a = nugen.fill(M, K, 5, nugen.MAT_A, kind)
    b = nugen.fill(K, N, 5, nugen.MAT_B, kind)
    ref = oracle.gemm(a, b)
    if kind == "int":
        assert np.array_equal(Cs[0].astype(np.float64), ref)
    else:
        e, where = oracle.normwise_err(Cs[0], ref, oracle.row_norms(a), oracle.col_norms(b))
        assert e <= 1e-5, (e, where)


def test_multiprocess_dead_peer_fails_loudly(tmp_path):
    """A sibling process that never runs its part: the other sibling's call
    returns NU_ECUDA after NORTHUP_PEER_TIMEOUT_S instead of blocking forever
    on the device-side flag waits."""
    env = dict(os.environ, PEER_SKIP_GEMM="1", NORTHUP_PEER_TIMEOUT_S="5")
    d, procs = spawn(tmp_path, 2, 512, 512, 1024, 256, 0, "int", 1, env=env)
    outs = []
    try:
        for p in procs:
            out, _ = p.communicate(timeout=180)
            outs.append(out.decode(errors="replace"))
    finally:
        for p in procs:
            if p.poll() is None:
                p.kill()
    assert procs[0].returncode == 3, outs[0]
    assert "no progress from the peer processes" in outs[0]
    assert procs[1].returncode == 0, outs[1]
