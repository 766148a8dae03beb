import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
sys.path.insert(0, "tests")
import numpy as np, torch
import nugen, oracle
import paper_conf_ipps_chey19_b200 as nu
from test_gpu_tree import run_host
for (M, N, K, G, cap) in [(900, 900, 1024, 3, 4 << 20), (300, 900, 1024, 1, 4 << 20), (300, 900, 1024, 1, 4 << 20),
                          (300, 512, 1024, 1, 4 << 20), (256, 900, 1024, 1, 4 << 20), (300, 900, 512, 1, 4 << 20)]:
    Cs, a, b, ss = run_host(M, N, K, G=G, cap=cap, kind="int", seed=6, k_chunk=512, schedule=nu.NU_SCHED_S2)
    ref = oracle.gemm(a, b)
    d = np.argwhere(Cs.astype(np.float64) != ref)
    print((M, N, K, G), {k: ss[k] for k in ("bm", "bn", "tail_k", "strips")}, "ndiff", len(d),
          "rows", (d[:, 0].min(), d[:, 0].max()) if len(d) else None, "cols", np.unique(d[:, 1])[:10] if len(d) else None, flush=True)
