"""In-HBM leaf timing for one kernel variant (env NORTHUP_LEAF), CUDA events,
k_chunk 2048 (the product setting).  SZS: comma list of cube sizes."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chey19_b200 as nu

dev = torch.device("cuda:0")
KC = int(os.environ.get("KC", "2048"))
res = {"variant": os.environ.get("NORTHUP_LEAF", "default"), "k_chunk": KC}
for SZ in [int(s) for s in os.environ.get("SZS", "8192,16384").split(",")]:
    A = torch.rand((SZ, SZ), device=dev) * 2 - 1
    B = torch.rand((SZ, SZ), device=dev) * 2 - 1
    C = torch.empty((SZ, SZ), device=dev)
    it = 10 if SZ <= 16384 else 3
    for _ in range(2):
        nu.leaf_gemm(A, B, C, k_chunk=KC)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(it):
        nu.leaf_gemm(A, B, C, k_chunk=KC)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / it
    res[str(SZ)] = {"ms": round(ms, 3), "tflops": round(2 * SZ ** 3 / ms / 1e9, 1)}
    del A, B, C
print(json.dumps(res))
