"""Profile mode of the 2sm leaf: per-cluster cycles (total, MMA waiting on the
split, MMA waiting on the epilogue, k-blocks; split waiting on TMA / lo slot)."""
import ctypes, sys, os, json
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import paper_conf_ipps_chey19_b200 as nu
L = nu.lib(); f = L.northup_debug_leaf_gemm
f.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
              ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
              ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p]
dev = torch.device("cuda:0")
for SZ in [8192]:
    A = torch.rand((SZ, SZ), device=dev) - 0.5; B = torch.rand((SZ, SZ), device=dev) - 0.5
    C = torch.empty((SZ, SZ), device=dev); dbg = torch.zeros(8 * 80, device=dev)
    for npass, exp in ((2, 0),):
        for _ in range(2):
            rc = f(A.data_ptr(), SZ, B.data_ptr(), SZ, C.data_ptr(), SZ, SZ, SZ, SZ, 0, 2048, npass, exp, dbg.data_ptr(), int(os.environ.get("LEAF_VARIANT", "2")), None)
            assert rc == 0, nu.last_error()
        torch.cuda.synchronize()
        d = dbg.cpu().numpy().reshape(80, 8)[:74]
        tot, wx, wt, kb = d[:, 0], d[:, 1], d[:, 2], d[:, 3]
        print(json.dumps({"SZ": SZ, "npass": npass, "exp": exp, "cycles_total_mean": float(tot.mean()),
              "mma_wait_split_frac": float((wx / tot).mean()), "mma_wait_epi_frac": float((wt / tot).mean()),
              "kblocks_per_cluster": float(kb.mean()),
              "cycles_per_kblock": float((tot / kb).mean()),
              "split_wait_tma_frac_leader": float((d[:, 4] / tot).mean()), "split_wait_loslot_frac_leader": float((d[:, 5] / tot).mean()),
              "split_wait_tma_frac_peer": float((d[:, 6] / tot).mean()), "split_wait_loslot_frac_peer": float((d[:, 7] / tot).mean())}))
