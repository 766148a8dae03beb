"""GPU check of the x3 leaf (split operands, fp16 x3): parity, adversarial
accuracy and speed.  Writes gpurun_out/x3_check.json.  (The round-2 sweep of the
TMEM accumulation chunk, profiles/r02/x3_check_acc{128,256,512}.json, ran with a
build-time knob since removed; the product chunk is kAccChunk = 256.)"""
import ctypes
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import torch

import nugen
import oracle
import paper_conf_ipps_chey19_b200 as nu

dev = torch.device("cuda:0")
f = nu.lib().northup_debug_leaf_gemm
f.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
              ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
              ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int,
              ctypes.c_void_p]
out = {}


def run(A, B, C=None, npass=0, kc=0, variant=0, acc=0, ldc_pad=0):
    M, K = A.shape
    N = B.shape[1]
    if C is None:
        C = torch.full((M, N + ldc_pad), float("nan"), device=dev)
    rc = f(A.data_ptr(), A.stride(0), B.data_ptr(), B.stride(0), C.data_ptr(), C.stride(0), M, N, K, acc, kc,
           npass, 0, None, variant, torch.cuda.current_stream().cuda_stream)
    if rc != 0:
        raise RuntimeError(nu.last_error())
    torch.cuda.synchronize()
    return C


def nw(C, A, B):
    Ad, Bd = A.double().cpu(), B.double().cpu()
    ref = Ad @ Bd
    den = Ad.norm(dim=1)[:, None] * Bd.norm(dim=0)[None, :]
    d = (C[:, :B.shape[1]].double().cpu() - ref)
    e = d.abs() / den
    z = den == 0
    e[z] = torch.where(d[z] == 0, torch.zeros_like(d[z]), torch.full_like(d[z], float("inf")))
    return float(e.max())


try:
    # integer inputs: exact
    for (M, N, K) in [(256, 256, 32), (1, 1, 1), (257, 300, 65), (33, 17, 40), (512, 768, 1024),
                      (1000, 1000, 999), (384, 768, 2056), (300, 260, 4100)]:
        A = torch.from_numpy(nugen.fill(M, K, 11, 1, "int")).to(dev)
        B = torch.from_numpy(nugen.fill(K, N, 11, 2, "int")).to(dev)
        C = run(A, B)
        ref = A.double().cpu() @ B.double().cpu()
        out[f"int_{M}x{N}x{K}"] = bool(torch.equal(C.double().cpu(), ref))
        Cu = run(A, B, ldc_pad=1)   # unaligned-ld C: register epilogue
        out[f"int_{M}x{N}x{K}_ldc+1"] = bool(torch.equal(Cu[:, :N].double().cpu(), ref)) and bool(
            torch.isnan(Cu[:, N:]).all())
    for (M, N, K) in [(128, 256, 32), (257, 300, 65), (1000, 1000, 999), (512, 512, 2048), (300, 520, 3000)]:
        A = torch.from_numpy(nugen.fill(M, K, 12, 1)).to(dev)
        B = torch.from_numpy(nugen.fill(K, N, 12, 2)).to(dev)
        for npass in (1, 3, 4):
            out[f"uni_{M}x{N}x{K}_np{npass}"] = nw(run(A, B, npass=npass), A, B)
    # accumulate
    A = torch.from_numpy(nugen.fill(300, 3000, 14, 1)).to(dev)
    B = torch.from_numpy(nugen.fill(3000, 520, 14, 2)).to(dev)
    C0 = torch.from_numpy(nugen.fill(300, 520, 14, 3)).to(dev)
    C = C0.clone()
    run(A, B, C=C, acc=1)
    ref = A.double().cpu() @ B.double().cpu() + C0.double().cpu()
    den = A.double().cpu().norm(dim=1)[:, None] * B.double().cpu().norm(dim=0)[None, :]
    out["accumulate"] = float(((C.double().cpu() - ref).abs() / den).max())
    print(json.dumps(out), flush=True)
    # adversarial, several accumulation chunks (env read once per process: run chunks in sub-procs)
except Exception as e:  # noqa
    out["error"] = repr(e)
    print(json.dumps(out), flush=True)

acc_chunk = 256
adv = {}
M = N = 512
for c in (1.0048771, 0.3, 0.1256096, 1.0):
    for K in (2048, 32768):
        A = torch.full((M, K), c, device=dev)
        B = torch.full((K, N), c, device=dev)
        adv[f"const{c}_K{K}"] = nw(run(A, B), A, B)
g = torch.Generator(device=dev).manual_seed(7)
for K in (2048, 32768):
    A = torch.rand((M, K), device=dev, generator=g)
    B = torch.rand((K, N), device=dev, generator=g)
    adv[f"u01_K{K}"] = nw(run(A, B), A, B)
    A = torch.rand((M, K), device=dev, generator=g) * 2 - 1
    B = torch.rand((K, N), device=dev, generator=g) * 2 - 1
    adv[f"u11_K{K}"] = nw(run(A, B), A, B)
# row/column scaling: rows of A spanning 2^-40 .. 2^40
K = 4096
A = torch.rand((M, K), device=dev, generator=g) * 2 - 1
A *= torch.pow(2.0, torch.linspace(-40, 40, M, device=dev))[:, None]
B = torch.rand((K, N), device=dev, generator=g) * 2 - 1
B *= torch.pow(2.0, torch.linspace(30, -30, N, device=dev))[None, :]
adv["rowcol_scaled"] = nw(run(A, B), A, B)
out[f"adversarial_acc{acc_chunk}"] = adv
print(json.dumps(adv), flush=True)

perf = {}
for SZ in (8192, 32768):
    A = torch.rand((SZ, SZ), device=dev) * 2 - 1
    B = torch.rand((SZ, SZ), device=dev) * 2 - 1
    C = torch.empty((SZ, SZ), device=dev)
    for variant in (0,):
        reps = 5 if SZ == 8192 else 2
        run(A, B, C=C, variant=variant)
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(reps):
            f(A.data_ptr(), SZ, B.data_ptr(), SZ, C.data_ptr(), SZ, SZ, SZ, SZ, 0, 0, 0, 0, None, variant,
              torch.cuda.current_stream().cuda_stream)
        e1.record()
        torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / reps
        perf[f"{SZ}_v{variant}"] = {"ms": ms, "tflops": 2 * SZ ** 3 / ms / 1e9}
    print(json.dumps(perf), flush=True)
out[f"perf_acc{acc_chunk}"] = perf
os.makedirs("gpurun_out", exist_ok=True)
with open("gpurun_out/x3_check.json", "w") as fh:
    json.dump(out, fh, indent=1)
