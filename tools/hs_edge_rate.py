"""HotSpot leaf: one launch of 8 iterations on a 8704 x 8448 window placed in
the grid's interior, at its top edge, at its left edge and in its corner (the
out-of-core plan's window placements).  ms per launch."""
import json, os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chey19_b200 as nu

R = C = 32768
WM, WN = 8704, 8448
t = torch.rand(WM, WN, device="cuda") * 10 + 330
p = torch.rand(WM, WN, device="cuda") * 0.5
o = torch.empty_like(t)
res = {}
for name, gy, gx in [("interior", 8000, 8000), ("top", 0, 8000), ("left", 8000, 0), ("right", 8000, C - WN),
                     ("corner", 0, 0)]:
    for _ in range(3):
        nu.hotspot_leaf(t, p, o, 8, gy0=gy, gx0=gx, rows=R, cols=C)
    torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(30):
        nu.hotspot_leaf(t, p, o, 8, gy0=gy, gx0=gx, rows=R, cols=C)
    e1.record()
    torch.cuda.synchronize()
    res[name] = round(e0.elapsed_time(e1) / 30, 4)
print(json.dumps(res), flush=True)
