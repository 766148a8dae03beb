"""Accuracy probe of the leaf on adversarial (same-sign) inputs, VERDICT r1 item 1.

Constant matrices A = B = c.1 make every product err with the same sign, so the
normwise error equals the per-product split error plus the accumulation bias.
Also probes the tensor core's accumulator rounding with exactly representable
inputs: row a = [1, d, d, ...], B = ones, exact sum 1 + (K-1) d.
"""
import json
import os
import sys

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import ctypes

import numpy as np
import torch

import paper_conf_ipps_chey19_b200 as nu

dev = torch.device("cuda:0")
L = nu.lib()
f = L.northup_debug_leaf_gemm
f.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
              ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
              ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
              ctypes.c_void_p]


def run(A, B, npass=0, kc=0, variant=0):
    M, K = A.shape
    N = B.shape[1]
    C = torch.full((M, N), float("nan"), device=dev)
    rc = f(A.data_ptr(), A.stride(0), B.data_ptr(), B.stride(0), C.data_ptr(), N, M, N, K, 0, kc, npass, 0,
           None, variant, torch.cuda.current_stream().cuda_stream)
    assert rc == 0, nu.last_error()
    torch.cuda.synchronize()
    return C.double().cpu()


def normwise(C, A, B):
    Ad, Bd = A.double().cpu(), B.double().cpu()
    ref = Ad @ Bd
    den = Ad.norm(dim=1)[:, None] * Bd.norm(dim=0)[None, :]
    e = (C - ref).abs() / den
    return float(e.max()), float(((C - ref) / den).mean())


out = {}
variants = [("v3_np2", 2, 4), ("v12_np3", 3, 2)]
M = N = 512
for c in (1.0048771, 0.3, 1.0, 0.1256096):
    for K in (2048, 32768):
        A = torch.full((M, K), c, device=dev)
        B = torch.full((K, N), c, device=dev)
        for name, npass, var in variants:
            for kc in (2048, 512, 128):
                C = run(A, B, npass, kc, var)
                out[f"const{c}_K{K}_{name}_kc{kc}"] = normwise(C, A, B)
g = torch.Generator(device=dev).manual_seed(7)
for K in (2048, 32768):
    A = torch.rand((M, K), device=dev, generator=g)
    B = torch.rand((K, N), device=dev, generator=g)
    for name, npass, var in variants:
        for kc in (2048, 512, 128):
            out[f"u01_K{K}_{name}_kc{kc}"] = normwise(run(A, B, npass, kc, var), A, B)
    A = torch.rand((M, K), device=dev, generator=g) * 2 - 1
    B = torch.rand((K, N), device=dev, generator=g) * 2 - 1
    for name, npass, var in variants:
        out[f"u11_K{K}_{name}_kc2048"] = normwise(run(A, B, npass, 2048, var), A, B)
print(json.dumps(out, indent=1), flush=True)

# accumulator rounding: a = [1, d, d, ...] (exact in tf32, lo = 0), B = ones
acc = {}
for d_name, d in (("2^-24", 2.0 ** -24), ("2^-25", 2.0 ** -25), ("3*2^-25", 3 * 2.0 ** -25),
                  ("2^-22", 2.0 ** -22), ("-2^-24", -(2.0 ** -24))):
    for K in (8, 16, 32, 64, 256, 2048):
        A = torch.full((128, K), d, device=dev)
        A[:, 0] = 1.0
        B = torch.ones((K, 128), device=dev)
        for name, npass, var in variants:
            C = run(A, B, npass, 0, var)
            got = float(C[0, 0])
            exact = 1.0 + (K - 1) * d
            acc[f"a0=1_d={d_name}_K{K}_{name}"] = {"got_minus_1_in_2^-23": (got - 1.0) * 2 ** 23,
                                                   "exact_minus_1_in_2^-23": (exact - 1.0) * 2 ** 23}
    # tiny terms first, the large one last
    for K in (16, 256):
        A = torch.full((128, K), d, device=dev)
        A[:, K - 1] = 1.0
        B = torch.ones((K, 128), device=dev)
        for name, npass, var in variants:
            C = run(A, B, npass, 0, var)
            acc[f"last=1_d={d_name}_K{K}_{name}"] = {"got_minus_1_in_2^-23": (float(C[0, 0]) - 1.0) * 2 ** 23,
                                                     "exact_minus_1_in_2^-23": (K - 1) * d * 2 ** 23}
print(json.dumps(acc, indent=1), flush=True)
os.makedirs("gpurun_out", exist_ok=True)
with open("gpurun_out/acc_probe.json", "w") as fh:
    json.dump({"normwise": out, "accumulator": acc}, fh, indent=1)
