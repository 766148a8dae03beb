"""NEXT-2 on one B200: G virtual siblings, one of them slowed by the test
hook (NORTHUP_DEBUG_SLOW_SIBLING holds its compute stream before every leaf):
static S2 partition vs queue scheduling with stealing.  Also the symmetric
case (no slow sibling), where the queue's finer tiles cost PCIe bytes."""
import ctypes, json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import nugen
import paper_conf_ipps_chey19_b200 as nu

M = N = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
K = int(sys.argv[2]) if len(sys.argv) > 2 else 16384
G = 2
res = {"M": M, "N": N, "K": K, "G": G}
t, _ = nu.host_tree(G, 8 << 30, devices=[0] * G)
t.finalize()
A, B, C = t.alloc(4 * M * K, 0), t.alloc(4 * K * N, 0), t.alloc(4 * M * N, 0)
view = lambda b, r, c: np.ctypeslib.as_array((ctypes.c_float * (r * c)).from_address(b.ptr)).reshape(r, c)
nugen.fill(M, K, 4, 1, out=view(A, M, K))
nugen.fill(K, N, 4, 2, out=view(B, K, N))
ref = None
for slow in ("", "1,300"):     # sibling 1 takes 4x as long per leaf
    os.environ["NORTHUP_DEBUG_SLOW_SIBLING"] = slow
    for name, sched, tiles in (("static_s2", nu.NU_SCHED_S2, 0), ("queue2", nu.NU_SCHED_QUEUE, 2),
                               ("queue8", nu.NU_SCHED_QUEUE, 8)):
        o = nu.make_opts(schedule=sched, shared_staging=-1, queue_tiles=tiles)
        t.gemm(A, B, C, M, N, K, o)
        ts = []
        for _ in range(2):
            t0 = time.perf_counter()
            st = t.gemm(A, B, C, M, N, K, o)
            ts.append((time.perf_counter() - t0) * 1e3)
        c = view(C, M, N).copy()
        ref = c if ref is None else ref
        key = f"{name}{'_slow_sibling' if slow else ''}"
        res[key] = {"ms": min(ts), "tflops": 2.0 * M * N * K / min(ts) / 1e9, "tasks": st["tasks"],
                    "stolen": st["tasks_stolen"], "h2d_gib": st["bytes_h2d"] / 2**30,
                    "bitwise_vs_first": bool(np.array_equal(c, ref))}
        print(key, res[key], flush=True)
t.destroy()
os.makedirs("gpurun_out", exist_ok=True)
json.dump(res, open("gpurun_out/queue_bench.json", "w"), indent=1)
