"""cfg1 (256^3, 64x64 blocks, HOST -> GPU leaf) latency with and without CUDA graphs."""
import ctypes, sys, os, json, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import nugen
import paper_conf_ipps_chey19_b200 as nu
res = {}
for name, (M, N, K, blk) in {"cfg1": (256, 256, 256, (64, 64, 64)), "1k": (1024, 1024, 1024, None)}.items():
    t, _ = nu.host_tree(1)
    if blk: t.set_block(0, *blk)
    t.finalize()
    A, B, C = t.alloc(4 * M * K, 0), t.alloc(4 * K * N, 0), t.alloc(4 * M * N, 0)
    arr = lambda b, r, c: np.ctypeslib.as_array((ctypes.c_float * (r * c)).from_address(b.ptr)).reshape(r, c)
    nugen.fill(M, K, 1, 1, out=arr(A, M, K)); nugen.fill(K, N, 1, 2, out=arr(B, K, N))
    for graph in (False, True):
        o = nu.make_opts(graph=graph)
        for _ in range(5): t.gemm(A, B, C, M, N, K, o)
        n = 50
        t0 = time.perf_counter()
        for _ in range(n): st = t.gemm(A, B, C, M, N, K, o)
        res[f"{name}_graph{int(graph)}_ms"] = (time.perf_counter() - t0) / n * 1e3
        res[f"{name}_graph{int(graph)}_replayed"] = st["graph_replayed"]
        res[f"{name}_ops"] = st["ops"]
    t.destroy()
print(json.dumps(res, indent=1))
