import ctypes, sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import paper_conf_ipps_chey19_b200 as nu
L = nu.lib(); f = L.northup_debug_mma_rate
f.argtypes = [ctypes.c_int, ctypes.c_int, ctypes.c_int, ctypes.c_void_p]
out = torch.zeros(1, dtype=torch.int64, device="cuda")
for grid in (2, 148):
    for mode in (0, 1, 3):
        n = 3000
        for _ in range(2):
            assert f(n, mode, grid, out.data_ptr()) == 0, nu.last_error()
        print(json.dumps({"grid": grid, "mode": mode, "cycles_per_mma": out.item() / n}))
