"""Small runs for compute-sanitizer (memcheck / racecheck / synccheck)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch, ctypes
import nugen
import paper_conf_ipps_chey19_b200 as nu
dev = torch.device("cuda:0")
for (M, N, K, npass) in [(300, 300, 132, 2), (256, 512, 96, 3), (130, 72, 40, 2)]:
    A = torch.from_numpy(nugen.fill(M, K, 1, 1)).to(dev)
    B = torch.from_numpy(nugen.fill(K, N, 1, 2)).to(dev)
    C = torch.empty((M, N), device=dev)
    nu.leaf_gemm(A, B, C, npass=npass, k_chunk=64)
torch.cuda.synchronize()
t, _ = nu.host_tree(2, devices=[0, 0])
t.finalize()
M, N, K = 300, 260, 200
Ab, Bb, Cb = t.alloc(4 * M * K, 0), t.alloc(4 * K * N, 0), t.alloc(4 * M * N, 0)
a = np.ctypeslib.as_array((ctypes.c_float * (M * K)).from_address(Ab.ptr)).reshape(M, K)
b = np.ctypeslib.as_array((ctypes.c_float * (K * N)).from_address(Bb.ptr)).reshape(K, N)
nugen.fill(M, K, 1, 1, out=a); nugen.fill(K, N, 1, 2, out=b)
t.gemm(Ab, Bb, Cb, M, N, K, nu.make_opts(k_chunk=64))
t.destroy()
print("sanitize run ok")
