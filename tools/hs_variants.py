"""HotSpot leaf variants (NORTHUP_HS_LEAF) on a resident 16384^2 grid, 64
iterations at 8 per launch: GCUPS and bitwise equality with variant 3."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import nugen
import paper_conf_ipps_chey19_b200 as nu
R = C = int(os.environ.get("HS_N", "16384"))
IT = 64
T = torch.from_numpy(nugen.fill(R, C, 7, nugen.MAT_T, "temp")).cuda()
P = torch.from_numpy(nugen.fill(R, C, 7, nugen.MAT_P, "power")).cuda()
th = nu.hbm_tree(0); th.finalize()
O = torch.empty_like(T)
hT, hP, hO = (th.wrap_device(0, x.data_ptr(), x.numel() * 4) for x in (T, P, O))
out = {}
ref = None
for v in os.environ.get("HS_VARIANTS", "3,5").split(","):
    os.environ["NORTHUP_HS_LEAF"] = v
    th.hotspot(hT, hP, hO, R, C, IT, nu.hotspot_opts(leaf_iters=8)); torch.cuda.synchronize()
    res = O.clone()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3):
        th.hotspot(hT, hP, hO, R, C, IT, nu.hotspot_opts(leaf_iters=8))
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1) / 3
    if ref is None:
        ref = res
    out[v] = {"gcups": R * C * IT / ms / 1e6, "bitwise_vs_first": bool(torch.equal(res, ref))}
print(json.dumps(out), flush=True)
