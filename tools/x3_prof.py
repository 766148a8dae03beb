"""Profile mode of the x3 leaf: the MMA issuer's cycle counters (dbg buffer) on one
K panel (32768 x 32768 x 2048 by default), plus CUDA-event timing of split and GEMM."""
import ctypes
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch

import paper_conf_ipps_chey19_b200 as nu

dev = torch.device("cuda:0")
f = nu.lib().northup_debug_leaf_gemm
f.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
              ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
              ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
              ctypes.c_void_p]
M = N = int(os.environ.get("SZ", "32768"))
K = int(os.environ.get("KK", "2048"))
A = torch.rand((M, K), device=dev) * 2 - 1
B = torch.rand((K, N), device=dev) * 2 - 1
C = torch.empty((M, N), device=dev)
dbg = torch.zeros(4 * 80, device=dev)
s = torch.cuda.current_stream().cuda_stream
for _ in range(3):
    assert f(A.data_ptr(), K, B.data_ptr(), N, C.data_ptr(), N, M, N, K, 0, 0, 0, 0, None, 0, s) == 0
torch.cuda.synchronize()
e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
e0.record()
for _ in range(5):
    f(A.data_ptr(), K, B.data_ptr(), N, C.data_ptr(), N, M, N, K, 0, 0, 0, 0, None, 0, s)
e1.record()
torch.cuda.synchronize()
ms = e0.elapsed_time(e1) / 5
f(A.data_ptr(), K, B.data_ptr(), N, C.data_ptr(), N, M, N, K, 0, 0, 0, 0, dbg.data_ptr(), 0, s)
torch.cuda.synchronize()
d = dbg.view(-1, 4).cpu()
d = d[d[:, 3] > 0]
tot, wf, wt, st = d.sum(0).tolist()
res = {"M": M, "N": N, "K": K, "ms_per_call": ms, "tflops_incl_split": 2 * M * N * K / ms / 1e9,
       "clusters": len(d), "clk_per_stage": tot / st, "mma_wait_full_pct": 100 * wf / tot,
       "mma_wait_tempty_pct": 100 * wt / tot}
print(json.dumps(res), flush=True)
