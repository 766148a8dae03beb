"""Small runs of the round's newer paths for compute-sanitizer: the HotSpot
leaf variants (v1/v2/v3 via NORTHUP_HS_LEAF), the HotSpot tree (HOST root,
2 virtual siblings), shared staging (2 virtual siblings) and the queue
schedule with a slow sibling."""
import ctypes, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import nugen
import paper_conf_ipps_chey19_b200 as nu

dev = torch.device("cuda:0")
R, C = 150, 300
T = torch.from_numpy(nugen.fill(R, C, 1, nugen.MAT_T, "temp")).to(dev)
P = torch.from_numpy(nugen.fill(R, C, 1, nugen.MAT_P, "power")).to(dev)
O = torch.empty_like(T)
for it in (1, 5, 8):
    nu.hotspot_leaf(T, P, O, it)
    nu.hotspot_leaf(T[20:120, 30:250].contiguous(), P[20:120, 30:250].contiguous(),
                    torch.empty((100, 220), device=dev), it, gy0=20, gx0=30, rows=R, cols=C)
torch.cuda.synchronize()
view = lambda b, r, c: np.ctypeslib.as_array((ctypes.c_float * (r * c)).from_address(b.ptr)).reshape(r, c)
t, _ = nu.host_tree(2, devices=[0, 0])
t.finalize()
Tb, Pb, Ob = t.alloc(4 * R * C, 0), t.alloc(4 * R * C, 0), t.alloc(4 * R * C, 0)
view(Tb, R, C)[...] = T.cpu().numpy()
view(Pb, R, C)[...] = P.cpu().numpy()
t.hotspot(Tb, Pb, Ob, R, C, 11, nu.hotspot_opts(block=64, halo=4, leaf_iters=3))
M, N, K = 256, 192, 160
Ab, Bb, Cb = t.alloc(4 * M * K, 0), t.alloc(4 * K * N, 0), t.alloc(4 * M * N, 0)
nugen.fill(M, K, 1, 1, out=view(Ab, M, K))
nugen.fill(K, N, 1, 2, out=view(Bb, K, N))
st = t.gemm(Ab, Bb, Cb, M, N, K, nu.make_opts(k_chunk=64))
assert st["shared_staging"] == 1
os.environ["NORTHUP_DEBUG_SLOW_SIBLING"] = "1,200"
t.gemm(Ab, Bb, Cb, M, N, K, nu.make_opts(k_chunk=64, schedule=nu.NU_SCHED_QUEUE, queue_tiles=4))
t.destroy()
print("sanitize2 run ok")
