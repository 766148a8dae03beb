"""Out-of-core cfg3 timeline: per-stream busy time, fill/drain and compute gaps."""
import ctypes, sys, os, json, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import nugen
import paper_conf_ipps_chey19_b200 as nu
SZ = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
cap = (8 << 30) * (SZ // 32768) ** 2 if SZ >= 32768 else (8 << 30) // (32768 // SZ) ** 2
M = N = K = SZ
t, hbm = nu.host_tree(1, cap)
t.finalize()
A, B, C = t.alloc(4 * M * K, 0), t.alloc(4 * K * N, 0), t.alloc(4 * M * N, 0)
arr = lambda b, r, c: np.ctypeslib.as_array((ctypes.c_float * (r * c)).from_address(b.ptr)).reshape(r, c)
nugen.fill(M, K, 3, 1, out=arr(A, M, K)); nugen.fill(K, N, 3, 2, out=arr(B, K, N))
for _ in range(2):
    t.gemm(A, B, C, M, N, K)
st = t.gemm(A, B, C, M, N, K, nu.make_opts(collect_timing=True))
L = nu.lib(); f = L.northup_debug_timeline
f.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int]; f.restype = ctypes.c_int
buf = np.zeros(5 * 20000, dtype=np.float32)
n = f(t.handle, buf.ctypes.data, 20000)
tl = buf[: 5 * n].reshape(n, 5)
ops = t.plan(M, N, K).ops()
comp = tl[tl[:, 2] == 1]; h2d = tl[tl[:, 2] == 0]; d2h = tl[tl[:, 2] == 2]
comp = comp[np.argsort(comp[:, 3])]
gaps = np.maximum(0, comp[1:, 3] - comp[:-1, 4])
end = tl[:, 4].max()
res = {"total_ms": st["t_total_ms"], "timeline_end_ms": float(end),
       "first_compute_start_ms": float(comp[0, 3]), "last_compute_end_ms": float(comp[:, 4].max()),
       "drain_after_compute_ms": float(end - comp[:, 4].max()),
       "compute_busy_ms": float((comp[:, 4] - comp[:, 3]).sum()), "compute_gaps_ms": float(gaps.sum()),
       "largest_gaps_ms": [float(x) for x in sorted(gaps.tolist())[-5:]],
       "h2d_busy_ms": float((h2d[:, 4] - h2d[:, 3]).sum()), "d2h_busy_ms": float((d2h[:, 4] - d2h[:, 3]).sum()),
       "h2d_GBps": st["bytes_h2d"] / max(1e-9, (h2d[:, 4] - h2d[:, 3]).sum()) / 1e6,
       "d2h_GBps": st["bytes_d2h"] / max(1e-9, (d2h[:, 4] - d2h[:, 3]).sum()) / 1e6,
       "launches": int(len(comp))}
print(json.dumps(res, indent=1, default=float))

# Coarse utilisation profile: per 10 ms bucket, busy fraction of H2D / compute / D2H.
def busy_in(rows, a, b):
    return float(np.clip(np.minimum(b, rows[:, 4]) - np.maximum(a, rows[:, 3]), 0, None).sum()) / (b - a)

prof = []
for a in np.arange(0.0, end, 10.0):
    b = a + 10.0
    prof.append([round(float(a)), round(busy_in(h2d, a, b), 2), round(busy_in(comp, a, b), 2), round(busy_in(d2h, a, b), 2)])
print("bucket_ms h2d comp d2h")
for r in prof:
    print(*r)
print("first_d2h_start_ms", float(d2h[:, 3].min()) if len(d2h) else None, "last_h2d_end_ms", float(h2d[:, 4].max()))

# leaf ops: TF/s per op (2 m n k / duration), early ops vs strips
lr = []
for row in comp:
    op = ops[int(row[0])]
    if op["op"] == nu.NU_OP_LEAF:
        d = float(row[4] - row[3])
        lr.append((float(row[3]), op["m"], op["n"], op["k"], d, 2.0 * op["m"] * op["n"] * op["k"] / d / 1e9))
lr = np.array(lr)
if len(lr):
    for lab, sel in (("m>=8192", lr[:, 1] >= 8192), ("m<8192", lr[:, 1] < 8192)):
        if sel.any():
            x = lr[sel]
            print(lab, "ops", int(sel.sum()), "busy_ms", round(float(x[:, 4].sum()), 2),
                  "tflops_total", round(float((2 * x[:, 1] * x[:, 2] * x[:, 3]).sum() / x[:, 4].sum() / 1e9), 1),
                  "shape", x[0, 1:4].astype(int).tolist(), "rate_min/med/max",
                  [round(float(v), 1) for v in np.percentile(x[:, 5], [0, 50, 100])])
if len(lr):
    big_k = lr[lr[:, 3] >= 16384]
    print("strip ops (k >= 16384): start_ms m n k ms TF/s")
    for r in big_k:
        print(round(r[0], 1), int(r[1]), int(r[2]), int(r[3]), round(r[4], 2), round(r[5], 1))
