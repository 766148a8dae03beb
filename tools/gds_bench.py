"""NEXT-4 GDS edge on one B200: a GEMM whose A, B, C live in files, through
(a) FILE -> HOST staging -> HBM (DRAM bounce level in the tree),
(b) FILE -> HBM directly through the library's pinned bounce buffer (default),
    or with cuFile when NORTHUP_CUFILE=1 (compat mode on this pool's virtio disk).
A is preprocessed to the K-panel-major layout (R15, outside the timing)."""
import json, os, sys, time, tempfile
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import nugen
import oracle
import paper_conf_ipps_chey19_b200 as nu

M = N = K = int(sys.argv[1]) if len(sys.argv) > 1 else 16384
PANEL = 2048
d = tempfile.mkdtemp(dir=os.environ.get("GDS_DIR", "/tmp"))
A = nugen.fill(M, K, 9, 1)
B = nugen.fill(K, N, 9, 2)
A.tofile(f"{d}/A.bin"); B.tofile(f"{d}/B.bin")
nu.file_tile_kpanels(f"{d}/A.bin", f"{d}/A_t.bin", M, K, PANEL)
res = {"M": M, "N": N, "K": K, "panel": PANEL, "dir": d}


def tree(kind):
    t = nu.Tree()
    root = t.add_node(-1, nu.NU_FILE)
    parent = t.add_node(root, nu.NU_HOST, -1, 0) if kind == "staging" else root
    h = t.add_node(parent, nu.NU_HBM, 0, 8 << 30)
    t.add_node(h, nu.NU_SMEM, 0, 227 * 1024, nu.NU_PROC_SM100)
    return t


# cuFile is opt-in (NORTHUP_CUFILE=1, read once per process): with it set the
# direct leg runs through cuFile, else through the pinned bounce buffer
direct = "direct_cufile" if os.environ.get("NORTHUP_CUFILE") == "1" else "direct_bounce"
for kind in ("staging", direct):
    t = tree("staging" if kind == "staging" else "direct")
    t.finalize()
    fa = t.open_file(0, f"{d}/A_t.bin", 4 * M * K)
    fb = t.open_file(0, f"{d}/B.bin", 4 * K * N)
    fc = t.open_file(0, f"{d}/C_{kind}.bin", 4 * M * N)
    o = nu.make_opts(a_panel_k=PANEL)
    t.gemm(fa, fb, fc, M, N, K, o)
    ms = []
    for _ in range(2):
        t0 = time.perf_counter()
        st = t.gemm(fa, fb, fc, M, N, K, o)
        ms.append((time.perf_counter() - t0) * 1e3)
    t.destroy()
    C = np.fromfile(f"{d}/C_{kind}.bin", dtype=np.float32).reshape(M, N)
    rows = np.arange(0, M, M // 16)
    ref = oracle.gemm_rows(A, B, rows)
    e, _ = oracle.normwise_err(np.ascontiguousarray(C[rows]), ref, oracle.row_norms(np.ascontiguousarray(A[rows])),
                               oracle.col_norms(B))
    res[kind] = {"ms": min(ms), "tflops": 2.0 * M * N * K / min(ms) / 1e9,
                 "file_read_gib": st["bytes_file_read"] / 2**30, "file_write_gib": st["bytes_file_write"] / 2**30,
                 "io_ms": st["t_io_ms"], "file_direct_mode": st["file_direct_mode"],
                 "normwise_err_16_rows": e}
    print(kind, res[kind], flush=True)
os.makedirs("gpurun_out", exist_ok=True)
json.dump(res, open("gpurun_out/gds_bench.json", "w"), indent=1)
