import os, sys, json, subprocess
sys.path.insert(0, "/root/repo"); sys.path.insert(0, "/root/repo/tests")
case = sys.argv[1]
import numpy as np
from test_gpu_hotspot import run_tree, emulate_fp32
G, li, block, halo = [int(x) for x in case.split(",")]
try:
    out, T, P, st = run_tree(1000, 1200, 20, G, 0, block=block, halo=halo, leaf_iters=li)
    print(case, "ok", bool(np.array_equal(out, emulate_fp32(T, P, 20))))
except Exception as e:
    print(case, "ERR", e)
