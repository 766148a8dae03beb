"""HotSpot-2D (NEXT-3) throughput on one B200: the in-HBM leaf at several
iterations per launch, and the HOST -> HBM out-of-core tree with a capped
HBM node.  Cell updates per second (GCUPS) = rows * cols * iters / time."""
import ctypes, json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import nugen
import paper_conf_ipps_chey19_b200 as nu

R = C = int(sys.argv[1]) if len(sys.argv) > 1 else 32768
ITERS = int(sys.argv[2]) if len(sys.argv) > 2 else 64
CAP = (int(sys.argv[3]) if len(sys.argv) > 3 else 8) << 30
dev = torch.device("cuda", 0)
res = {"R": R, "C": C, "iters": ITERS}
T = nugen.fill(R, C, 7, nugen.MAT_T, "temp")
P = nugen.fill(R, C, 7, nugen.MAT_P, "power")
Td, Pd = torch.from_numpy(T).to(dev), torch.from_numpy(P).to(dev)
Od = torch.empty_like(Td)
th = nu.hbm_tree(0)
th.finalize()
hT, hP, hO = (th.wrap_device(0, x.data_ptr(), x.numel() * 4) for x in (Td, Pd, Od))
for li in (1, 2, 4, 8):
    o = nu.hotspot_opts(leaf_iters=li)
    th.hotspot(hT, hP, hO, R, C, ITERS, o)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3):
        th.hotspot(hT, hP, hO, R, C, ITERS, o)
    e1.record()
    torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 3
    launches = -(-ITERS // li)
    res[f"in_hbm_leaf{li}"] = {"ms": ms, "gcups": R * C * ITERS / ms / 1e6,
                               "hbm_gbs_algorithmic": 12.0 * R * C * launches / ms / 1e6}
    print(li, res[f"in_hbm_leaf{li}"], flush=True)
ref = Od.cpu().numpy()
th.destroy()
if os.environ.get("HS_IN_HBM_ONLY"):
    print(json.dumps(res))
    sys.exit(0)
del Td, Pd, Od
torch.cuda.empty_cache()
t, _ = nu.host_tree(1, CAP)
t.finalize()
Tb, Pb, Ob = t.alloc(4 * R * C, 0), t.alloc(4 * R * C, 0), t.alloc(4 * R * C, 0)
view = lambda b: np.ctypeslib.as_array((ctypes.c_float * (R * C)).from_address(b.ptr)).reshape(R, C)
view(Tb)[...] = T
view(Pb)[...] = P
o = nu.hotspot_opts(block=int(os.environ.get("HS_BLOCK", "0")))
t.hotspot(Tb, Pb, Ob, R, C, ITERS, o)
ms = []
for _ in range(2):
    t0 = time.perf_counter()
    st = t.hotspot(Tb, Pb, Ob, R, C, ITERS, o)
    ms.append((time.perf_counter() - t0) * 1e3)
tim = t.hotspot(Tb, Pb, Ob, R, C, ITERS, nu.hotspot_opts(collect_timing=True))
res["ooc"] = {"ms": min(ms), "gcups": R * C * ITERS / min(ms) / 1e6, "block": st["bm"], "halo": st["bk"],
              "h2d_gib": st["bytes_h2d"] / 2**30, "d2h_gib": st["bytes_d2h"] / 2**30, "launches": st["leaf_launches"],
              "busy_ms": {"h2d": tim["t_h2d_ms"], "compute": tim["t_compute_ms"], "d2h": tim["t_d2h_ms"]},
              "bitwise_vs_in_hbm": bool(np.array_equal(view(Ob), ref))}
print(res["ooc"], flush=True)
t.destroy()
os.makedirs("gpurun_out", exist_ok=True)
json.dump(res, open("gpurun_out/hotspot_perf.json", "w"), indent=1)
