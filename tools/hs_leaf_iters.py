"""HotSpot-2D in-HBM GCUPS vs iterations per leaf launch (32768^2 grid, 240 iterations)."""
import sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, nugen
import paper_conf_ipps_chey19_b200 as nu
R = C = 32768; IT = 240
T = torch.from_numpy(nugen.fill(R, C, 7, nugen.MAT_T, "temp")).cuda()
P = torch.from_numpy(nugen.fill(R, C, 7, nugen.MAT_P, "power")).cuda()
O = torch.empty_like(T)
th = nu.hbm_tree(0); th.finalize()
hT, hP, hO = (th.wrap_device(0, x.data_ptr(), x.numel() * 4) for x in (T, P, O))
out = {}
for li in [int(v) for v in os.environ.get('LIS', '4,6,7,8').split(',')]:
    th.hotspot(hT, hP, hO, R, C, IT, nu.hotspot_opts(leaf_iters=li)); torch.cuda.synchronize()
    e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    e0.record()
    for _ in range(3):
        th.hotspot(hT, hP, hO, R, C, IT, nu.hotspot_opts(leaf_iters=li))
    e1.record(); torch.cuda.synchronize()
    out[li] = round(R * C * IT / (e0.elapsed_time(e1) / 3) / 1e6, 1)
print(json.dumps(out))
