import sys, os, ctypes, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import nugen, oracle
import paper_conf_ipps_chey19_b200 as nu
sys.path.insert(0, "tests")
from test_gpu_tree import run_host
M, N, K, G, cap = 900, 900, 1024, 3, 4 << 20
Cq, a, b, sq = run_host(M, N, K, G=G, cap=cap, kind="uniform", seed=6, k_chunk=512, schedule=nu.NU_SCHED_QUEUE)
Cs, _, _, ss = run_host(M, N, K, G=G, cap=cap, kind="uniform", seed=6, k_chunk=512, schedule=nu.NU_SCHED_S2)
d = np.argwhere(Cq != Cs)
print("ndiff", len(d), "rows", np.unique(d[:, 0])[:20], "cols", np.unique(d[:, 1])[:20])
print({k: sq[k] for k in ("bm", "bn", "bk", "tail_k", "tasks")}, {k: ss[k] for k in ("bm", "bn", "bk", "tail_k", "strips")})
Ad, Bd = torch.from_numpy(a).cuda(), torch.from_numpy(b).cuda()
Cl = torch.empty((M, N), device="cuda")
nu.leaf_gemm(Ad, Bd, Cl, k_chunk=512); torch.cuda.synchronize()
Cl = Cl.cpu().numpy()
print("leaf==queue", np.array_equal(Cl, Cq), "leaf==s2", np.array_equal(Cl, Cs))
dl = np.argwhere(Cl != Cs); print("leaf vs s2 diff rows", np.unique(dl[:, 0])[:30], len(dl))
rr = np.unique(dl[:, 0]); cc = np.unique(dl[:, 1])
print("rows", rr.min(), rr.max(), len(rr), "cols", cc)
ref = oracle.gemm(a, b)
rel = np.abs(Cs - ref)[dl[:, 0], dl[:, 1]] / (np.linalg.norm(a[dl[:, 0]].astype(np.float64), axis=1) * np.linalg.norm(b[:, dl[:, 1]].astype(np.float64), axis=0))
rl = np.abs(Cl - ref)[dl[:, 0], dl[:, 1]] / (np.linalg.norm(a[dl[:, 0]].astype(np.float64), axis=1) * np.linalg.norm(b[:, dl[:, 1]].astype(np.float64), axis=0))
print("s2 err at diffs max", rel.max(), "leaf err max", rl.max())
print("example", [(int(i), int(j), float(Cs[i, j]), float(Cl[i, j])) for i, j in dl[:4]])
