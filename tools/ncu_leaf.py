"""A few leaf launches for ncu (one shape, uniform inputs)."""
import sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chey19_b200 as nu
M = N = K = int(sys.argv[1]) if len(sys.argv) > 1 else 8192
dev = torch.device("cuda:0")
A = torch.rand((M, K), device=dev) * 2 - 1
B = torch.rand((K, N), device=dev) * 2 - 1
C = torch.empty((M, N), device=dev)
for _ in range(3):
    nu.leaf_gemm(A, B, C)
torch.cuda.synchronize()
print("done")
