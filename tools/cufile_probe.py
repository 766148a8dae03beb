"""Probe the opt-in cuFile path of the FILE -> HBM edge on a small GEMM (run
under `timeout`; NORTHUP_CUFILE_DEBUG prints each cuFile step to stderr)."""
import os, sys, tempfile
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
os.environ["NORTHUP_CUFILE"] = "1"
os.environ["NORTHUP_CUFILE_DEBUG"] = "1"
import numpy as np
import nugen
import paper_conf_ipps_chey19_b200 as nu
M = N = K = 512
d = tempfile.mkdtemp()
A = nugen.fill(M, K, 7, 1, "int"); B = nugen.fill(K, N, 7, 2, "int")
A.tofile(f"{d}/A.bin"); B.tofile(f"{d}/B.bin")
t = nu.Tree()
root = t.add_node(-1, nu.NU_FILE)
h = t.add_node(root, nu.NU_HBM, 0, 0)
t.add_node(h, nu.NU_SMEM, 0, 227 * 1024, nu.NU_PROC_SM100)
t.finalize()
fa = t.open_file(0, f"{d}/A.bin", 4 * M * K)
fb = t.open_file(0, f"{d}/B.bin", 4 * K * N)
fc = t.open_file(0, f"{d}/C.bin", 4 * M * N)
st = t.gemm(fa, fb, fc, M, N, K)
t.destroy()
C = np.fromfile(f"{d}/C.bin", dtype=np.float32).reshape(M, N)
print("mode", st["file_direct_mode"], "exact", np.array_equal(C.astype(np.float64), A.astype(np.float64) @ B), flush=True)
