"""Precision of the TMEM accumulation vs k_chunk (H3 probe) and leaf perf sweeps."""
import sys, os, json, subprocess, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import nugen, oracle
import paper_conf_ipps_chey19_b200 as nu
dev = torch.device("cuda:0")
mode = sys.argv[1] if len(sys.argv) > 1 else "all"
out = {}
if mode in ("all", "prec"):
    M, N, K = 256, 512, 32768
    A = nugen.fill(M, K, 3, 1); B = nugen.fill(K, N, 3, 2)
    ref = oracle.gemm(A, B); rn, cn = oracle.row_norms(A), oracle.col_norms(B)
    Ad, Bd = torch.from_numpy(A).to(dev), torch.from_numpy(B).to(dev)
    Cd = torch.empty((M, N), device=dev)
    for kc in [256, 1024, 2048, 4096, 8192, 32768]:
        nu.leaf_gemm(Ad, Bd, Cd, k_chunk=kc); torch.cuda.synchronize()
        e, _ = oracle.normwise_err(Cd.cpu().numpy(), ref, rn, cn)
        out[f"prec_K32768_kc{kc}"] = e
    # fp32 sequential round-to-nearest baseline for context (one column)
    print(json.dumps(out), flush=True)
if mode in ("all", "perf"):
    M = N = K = int(os.environ.get("SZ", "32768"))
    A = torch.rand((M, K), device=dev) * 2 - 1
    B = torch.rand((K, N), device=dev) * 2 - 1
    C = torch.empty((M, N), device=dev)
    for kc in [int(x) for x in os.environ.get("KCS", "1024,2048,4096").split(",")]:
        nu.leaf_gemm(A, B, C, k_chunk=kc); torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(3): nu.leaf_gemm(A, B, C, k_chunk=kc)
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 3
        out[f"perf_{M}_kc{kc}_band{os.environ.get('NORTHUP_RASTER_BAND','16')}_pan{os.environ.get('NORTHUP_PANEL_CHUNKS','1')}"] = round(2 * M * N * K / ms / 1e9, 1)
    print(json.dumps(out), flush=True)
