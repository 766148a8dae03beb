"""One in-HBM HotSpot sweep for ncu: 16384^2 grid, `iters` iterations with
`leaf_iters` per launch (the kernel under test is the leaf)."""
import os, sys
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch, nugen
import paper_conf_ipps_chey19_b200 as nu
R = C = int(os.environ.get("HS_N", "16384"))
li = int(sys.argv[1]) if len(sys.argv) > 1 else 8
T = torch.from_numpy(nugen.fill(R, C, 7, nugen.MAT_T, "temp")).cuda()
P = torch.from_numpy(nugen.fill(R, C, 7, nugen.MAT_P, "power")).cuda()
O = torch.empty_like(T)
th = nu.hbm_tree(0); th.finalize()
h = [th.wrap_device(0, x.data_ptr(), x.numel() * 4) for x in (T, P, O)]
for _ in range(2):
    th.hotspot(*h, R, C, 2 * li, nu.hotspot_opts(leaf_iters=li))
torch.cuda.synchronize()
th.destroy()
