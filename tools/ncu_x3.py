"""One in-HBM leaf call on 32768^2 x 4096 (two K-panel launches; the second
reduces into C, like 15 of the 16 panel launches of a cfg3 step).  Profile the
second GEMM kernel with: ncu -k regex:leaf_x3 -s 1 -c 1 ..."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chey19_b200 as nu
M = N = 32768
K = 4096
A = torch.rand((M, K), device="cuda") * 2 - 1
B = torch.rand((K, N), device="cuda") * 2 - 1
C = torch.empty((M, N), device="cuda")
nu.leaf_gemm(A, B, C)
torch.cuda.synchronize()
