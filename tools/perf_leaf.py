"""Quick leaf-kernel timing (in-HBM), CUDA events; context: cuBLAS fp32 / tf32."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chey19_b200 as nu

dev = torch.device("cuda:0")
res = {}
for (M, N, K, kc) in [(8192, 8192, 8192, 1024), (8192, 8192, 8192, 0), (16384, 16384, 8192, 1024)]:
    A = torch.rand((M, K), device=dev) * 2 - 1
    B = torch.rand((K, N), device=dev) * 2 - 1
    C = torch.empty((M, N), device=dev)
    for _ in range(3):
        nu.leaf_gemm(A, B, C, k_chunk=kc)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    it = 10
    e0.record()
    for _ in range(it):
        nu.leaf_gemm(A, B, C, k_chunk=kc)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / it
    res[f"leaf_{M}x{N}x{K}_kc{kc}"] = {"ms": ms, "tflops": 2 * M * N * K / ms / 1e9}
torch.backends.cuda.matmul.allow_tf32 = False
A = torch.rand((8192, 8192), device=dev); B = torch.rand((8192, 8192), device=dev)
for name, tf32 in [("cublas_fp32", False), ("cublas_tf32", True)]:
    torch.backends.cuda.matmul.allow_tf32 = tf32
    for _ in range(3): torch.matmul(A, B)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(10): torch.matmul(A, B)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 10
    res[name] = {"ms": ms, "tflops": 2 * 8192**3 / ms / 1e9}
print(json.dumps(res, indent=1))
