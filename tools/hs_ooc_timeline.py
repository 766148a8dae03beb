"""Out-of-core HotSpot timeline (32768^2 x 256, 8 GiB HBM cap): per-stream busy
time, compute gaps, and the leaf ops' cell-update rate against window size."""
import ctypes, json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import nugen
import paper_conf_ipps_chey19_b200 as nu

R = C = int(os.environ.get("HS_N", "32768"))
IT = int(os.environ.get("HS_IT", "256"))
cap = 8 << 30
t, _ = nu.host_tree(1, cap)
t.finalize()
Tb, Pb, Ob = t.alloc(4 * R * C, 0), t.alloc(4 * R * C, 0), t.alloc(4 * R * C, 0)
arr = lambda b: np.ctypeslib.as_array((ctypes.c_float * (R * C)).from_address(b.ptr)).reshape(R, C)
nugen.fill(R, C, 6, nugen.MAT_T, "temp", out=arr(Tb))
nugen.fill(R, C, 6, nugen.MAT_P, "power", out=arr(Pb))
for _ in range(2):
    st0 = t.hotspot(Tb, Pb, Ob, R, C, IT)
st = t.hotspot(Tb, Pb, Ob, R, C, IT, nu.hotspot_opts(collect_timing=1))
L = nu.lib(); f = L.northup_debug_timeline
f.argtypes = [ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int]; f.restype = ctypes.c_int
buf = np.zeros(5 * 50000, dtype=np.float32)
n = f(t.handle, buf.ctypes.data, 50000)
tl = buf[: 5 * n].reshape(n, 5)
ops = t.hotspot_plan(R, C, IT).ops()
comp = tl[tl[:, 2] == 1]
comp = comp[np.argsort(comp[:, 3])]
gaps = np.maximum(0, comp[1:, 3] - comp[:-1, 4])
rates = []
for row in comp:
    op = ops[int(row[0])]
    if op["op"] == nu.NU_OP_STENCIL:
        dur = row[4] - row[3]
        rates.append((op["m"], op["n"], op["k"], float(dur), op["m"] * op["n"] * op["k"] / max(dur, 1e-6) / 1e6))
rates.sort(key=lambda x: -x[3])
h2d = tl[tl[:, 2] == 0]; d2h = tl[tl[:, 2] == 2]
end = float(tl[:, 4].max())
res = {"step_ms_untimed": st0["t_total_ms"], "timeline_end_ms": end,
       "first_compute_start_ms": float(comp[0, 3]), "last_compute_end_ms": float(comp[:, 4].max()),
       "compute_busy_ms": float((comp[:, 4] - comp[:, 3]).sum()), "compute_gaps_ms": float(gaps.sum()),
       "largest_gaps_ms": [round(float(x), 3) for x in sorted(gaps.tolist())[-5:]],
       "h2d_busy_ms": float((h2d[:, 4] - h2d[:, 3]).sum()), "d2h_busy_ms": float((d2h[:, 4] - d2h[:, 3]).sum()),
       "h2d_first_start_ms": float(h2d[:, 3].min()), "h2d_last_end_ms": float(h2d[:, 4].max()),
       "stencil_ops": len(rates), "stencil_rows_m_n_k_ms_gcups_slowest": [tuple(round(v, 3) for v in r) for r in rates[:6]],
       "stencil_gcups_median": float(np.median([r[4] for r in rates])) if rates else None,
       "stats": {k: st[k] for k in ("bm", "bk", "leaf_launches", "bytes_h2d", "bytes_d2h")}}
print(json.dumps(res, indent=1, default=float))

# durations relative to the same-shape minimum, split by overlap with copies
def overlap(a0, a1, rows):
    return float(np.clip(np.minimum(a1, rows[:, 4]) - np.maximum(a0, rows[:, 3]), 0, None).sum())

byshape = {}
for row in comp:
    op = ops[int(row[0])]
    if op["op"] != nu.NU_OP_STENCIL:
        continue
    d = float(row[4] - row[3])
    byshape.setdefault((op["m"], op["n"]), []).append((d, overlap(row[3], row[4], h2d) / d, overlap(row[3], row[4], d2h) / d,
                                                      int(row[0])))
ratios = []
for k, v in byshape.items():
    mn = min(x[0] for x in v)
    for d, oh, od, i in v:
        ratios.append((d / mn, oh, od, i))
ratios = np.array(ratios)
if len(ratios):
    slow = ratios[ratios[:, 0] > 1.2]
    fast = ratios[ratios[:, 0] <= 1.05]
    print(json.dumps({"ops_with_shape_peers": len(ratios), "slow_over_1.2x": len(slow), "fast_within_5pct": len(fast),
                      "slow_mean_h2d_overlap": float(slow[:, 1].mean()) if len(slow) else None,
                      "slow_mean_d2h_overlap": float(slow[:, 2].mean()) if len(slow) else None,
                      "fast_mean_h2d_overlap": float(fast[:, 1].mean()) if len(fast) else None,
                      "fast_mean_d2h_overlap": float(fast[:, 2].mean()) if len(fast) else None,
                      "ratio_percentiles": [round(float(np.percentile(ratios[:, 0], q)), 3) for q in (10, 50, 90, 99)]},
                     indent=1))

# per leaf sequence (32 launches of one window): total busy and first window shape
seqs, cur = [], None
for row in comp:
    op = ops[int(row[0])]
    if op["op"] != nu.NU_OP_STENCIL:
        continue
    key = (op["src_off"], op["dst_off"]) if cur is None else None
    d = float(row[4] - row[3])
    if cur is None or op["m"] > cur["m_last"]:
        cur = {"gy0": op["src_off"], "gx0": op["dst_off"], "m0": op["m"], "n0": op["n"], "ms": 0.0, "launches": 0}
        seqs.append(cur)
    cur["ms"] += d
    cur["launches"] += 1
    cur["m_last"] = op["m"]
print(json.dumps([{k: (round(v, 3) if isinstance(v, float) else v) for k, v in s.items() if k != "m_last"}
                  for s in seqs]))
