"""Small runs of the round-2 paths for compute-sanitizer (memcheck / racecheck /
synccheck): the x3 leaf (split + GEMM) on ragged shapes, S2's B-first variant
(NU_SCHED_S2B, resident B split in place, strips), the persistent TMA HotSpot
leaf with several tiles per CTA (aligned, two launches on one stream: the
claimed-tile counter) and the v5 fallback (unaligned); replicate_result
pushes between two virtual siblings."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import nugen
import paper_conf_ipps_chey19_b200 as nu

dev = torch.device("cuda:0")
for (M, N, K) in [(300, 300, 132), (257, 520, 2100)]:
    A = torch.from_numpy(nugen.fill(M, K, 1, 1)).to(dev)
    B = torch.from_numpy(nugen.fill(K, N, 1, 2)).to(dev)
    C = torch.empty((M, N), device=dev)
    nu.leaf_gemm(A, B, C, k_chunk=512)
torch.cuda.synchronize()
t, _ = nu.host_tree(1, 0)
t.finalize()
M, N, K = 1100, 700, 900
a, b, c = t.alloc(4 * M * K, 0), t.alloc(4 * K * N, 0), t.alloc(4 * M * N, 0)
st = t.gemm(a, b, c, M, N, K, nu.make_opts(schedule=nu.NU_SCHED_S2B, k_chunk=256))
assert st["schedule"] == nu.NU_SCHED_S2B
t.destroy()
# replicate_result pushed by the plan (two virtual siblings on this device)
t, hbm = nu.host_tree(2, 0, devices=[0, 0])
t.finalize()
M, N, K = 700, 520, 300
reps = [torch.empty((M, N), device=dev) for _ in hbm]
for h, r in zip(hbm, reps):
    t.set_replica(h, r.data_ptr(), r.numel() * 4)
a, b, c = t.alloc(4 * M * K, 0), t.alloc(4 * K * N, 0), t.alloc(4 * M * N, 0)
st = t.gemm(a, b, c, M, N, K, nu.make_opts(replicate_result=True))
assert st["bytes_d2d"] >= 2 * 4 * M * N
t.destroy()
R, C_ = 2000, 1800
T = torch.from_numpy(nugen.fill(R, C_, 3, nugen.MAT_T, "temp")).to(dev)
P = torch.from_numpy(nugen.fill(R, C_, 3, nugen.MAT_P, "power")).to(dev)
O = torch.empty_like(T)
nu.hotspot_leaf(T, P, O, 7)                      # TMA kernel: 18 x 20 tiles over 148 CTAs
O2 = torch.empty_like(T)
nu.hotspot_leaf(O, P, O2, 8)                     # second launch on the stream: claimed-tile counter re-armed
buf = torch.empty(R * C_ + 4, device=dev)
Tu = buf[1:1 + R * C_].view(R, C_)
Tu.copy_(T)
nu.hotspot_leaf(Tu, P, O, 5)                     # unaligned base: v5
torch.cuda.synchronize()
print("sanitize_r2 ok")
