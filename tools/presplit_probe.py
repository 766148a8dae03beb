"""NU_LEAF2_PRESPLIT probe: C of a GEMM (uniform inputs, k_chunk 2048) saved to
gpurun_out/C_<tag>.npy for a bitwise comparison across leaf builds, plus timing."""
import os, sys, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import nugen
import paper_conf_ipps_chey19_b200 as nu
tag, M, N, K = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4])
dev = torch.device("cuda:0")
A = torch.from_numpy(nugen.fill(M, K, 5, 1)).to(dev)
B = torch.from_numpy(nugen.fill(K, N, 5, 2)).to(dev)
C = torch.empty((M, N), device=dev)
nu.leaf_gemm(A, B, C, k_chunk=2048)
torch.cuda.synchronize()
os.makedirs("gpurun_out", exist_ok=True)
np.save(f"gpurun_out/C_{tag}.npy", C.cpu().numpy())
for SZ in (8192, 32768):
    A2 = torch.rand((SZ, SZ), device=dev) * 2 - 1
    B2 = torch.rand((SZ, SZ), device=dev) * 2 - 1
    C2 = torch.empty((SZ, SZ), device=dev)
    for _ in range(2):
        nu.leaf_gemm(A2, B2, C2, k_chunk=2048)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    it = 10 if SZ == 8192 else 3
    e0.record()
    for _ in range(it):
        nu.leaf_gemm(A2, B2, C2, k_chunk=2048)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / it
    print(json.dumps({"tag": tag, "SZ": SZ, "ms": round(ms, 3), "tflops": round(2 * SZ ** 3 / ms / 1e9, 1)}))
    del A2, B2, C2
