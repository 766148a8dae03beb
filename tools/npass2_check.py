"""Quick parity + perf of the leaf with npass = 2 (tf32 hi.hi + bf16 cross) vs 3."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import nugen, oracle
import paper_conf_ipps_chey19_b200 as nu
dev = torch.device("cuda:0")
res = {}
for (M, N, K, kind) in [(256, 256, 32, "int"), (512, 768, 1024, "int"), (257, 300, 65, "int"),
                        (512, 512, 2048, "uniform"), (300, 520, 3000, "uniform"), (256, 512, 32768, "uniform")]:
    A = nugen.fill(M, K, 21, 1, kind); B = nugen.fill(K, N, 21, 2, kind)
    r4 = lambda x: -(-x // 4) * 4
    Ad = torch.zeros((M, r4(K)), device=dev); Ad[:, :K] = torch.from_numpy(A)
    Bd = torch.zeros((K, r4(N)), device=dev); Bd[:, :N] = torch.from_numpy(B)
    ref = oracle.gemm(A, B)
    for npass in (2, 3):
        Cd = torch.full((M, N), float("nan"), device=dev)
        nu.leaf_gemm(Ad[:, :K], Bd[:, :N], Cd, npass=npass); torch.cuda.synchronize()
        C = Cd.cpu().numpy()
        if kind == "int":
            res[f"{M}x{N}x{K}_{kind}_np{npass}"] = bool(np.array_equal(C.astype(np.float64), ref))
        else:
            res[f"{M}x{N}x{K}_{kind}_np{npass}"] = oracle.normwise_err(C, ref, oracle.row_norms(A), oracle.col_norms(B))[0]
print(json.dumps(res), flush=True)
for SZ in [int(x) for x in os.environ.get("SZS", "8192,32768").split(",")]:
    A = torch.rand((SZ, SZ), device=dev) * 2 - 1; B = torch.rand((SZ, SZ), device=dev) * 2 - 1
    C = torch.empty((SZ, SZ), device=dev)
    for npass in (2, 3):
        for _ in range(2): nu.leaf_gemm(A, B, C, npass=npass)
        torch.cuda.synchronize()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record()
        for _ in range(3): nu.leaf_gemm(A, B, C, npass=npass)
        e1.record(); torch.cuda.synchronize()
        ms = e0.elapsed_time(e1) / 3
        print(json.dumps({"SZ": SZ, "npass": npass, "tflops": 2 * SZ ** 3 / ms / 1e9}), flush=True)
