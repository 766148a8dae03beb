"""FILE root (S§8(a) a3): FILE -> HOST staging -> HBM -> SMEM/TMEM, with A in
the row-major or the K-panel-major (R15 preprocessed) file layout; C written
back to a file and checked against the fp64 oracle."""
import numpy as np
import pytest

import nugen
import oracle
import paper_conf_ipps_chey19_b200 as nu

pytestmark = pytest.mark.gpu


def file_tree(G, cap=0, staging_cap=0):
    t = nu.Tree()
    root = t.add_node(-1, nu.NU_FILE)
    st = t.add_node(root, nu.NU_HOST, -1, staging_cap)
    for g in range(G):
        h = t.add_node(st, nu.NU_HBM, 0, cap)
        t.add_node(h, nu.NU_SMEM, 0, 227 * 1024, nu.NU_PROC_SM100)
    return t


@pytest.mark.parametrize("M,N,K,G,cap,panel,kind", [
    (300, 200, 130, 1, 0, 0, "int"),
    (512, 768, 1024, 1, 0, 256, "uniform"),
    (640, 900, 1500, 2, 0, 512, "uniform"),
    (1000, 1200, 3000, 2, 8_000_000, 1024, "int"),      # capacity -> several C-block rounds
])
def test_file_root_gemm(tmp_path, M, N, K, G, cap, panel, kind):
    A = nugen.fill(M, K, 6, 1, kind)
    B = nugen.fill(K, N, 6, 2, kind)
    a_path, b_path, c_path = tmp_path / "A.bin", tmp_path / "B.bin", tmp_path / "C.bin"
    A.tofile(a_path)
    B.tofile(b_path)
    if panel:
        nu.file_tile_kpanels(str(a_path), str(tmp_path / "A_t.bin"), M, K, panel)
        a_path = tmp_path / "A_t.bin"
    t = file_tree(G, cap)
    t.finalize()
    fa = t.open_file(0, str(a_path), 4 * M * K)
    fb = t.open_file(0, str(b_path), 4 * K * N)
    fc = t.open_file(0, str(c_path), 4 * M * N)
    st = t.gemm(fa, fb, fc, M, N, K, nu.make_opts(a_panel_k=panel))
    t.destroy()
    C = np.fromfile(c_path, dtype=np.float32).reshape(M, N)
    ref = oracle.gemm(A, B)
    if kind == "int":
        assert np.array_equal(C.astype(np.float64), ref)
    else:
        e, _ = oracle.normwise_err(C, ref, oracle.row_norms(A), oracle.col_norms(B))
        assert e <= 1e-5, e
    assert st["bytes_file_write"] == 4 * M * N and st["bytes_file_read"] >= 4 * (M * K + K * N)


def test_file_alloc_and_move(tmp_path):
    """Table I alloc() at a FILE node creates a file; move_data
    file <-> host round-trips bytes; destroy removes the created file."""
    t = file_tree(1)
    t.set_file_dir(str(tmp_path))
    t.finalize()
    f = t.alloc(1 << 16, 0)
    h = t.alloc(1 << 16, 1)
    back = t.alloc(1 << 16, 1)
    import ctypes
    x = np.ctypeslib.as_array((ctypes.c_float * (1 << 14)).from_address(h.ptr))
    x[:] = nugen.fill(1, 1 << 14, 3, 1)[0]
    t.move_data(f, 0, h, 0, 1 << 16)
    t.move_data(back, 0, f, 0, 1 << 16)
    y = np.ctypeslib.as_array((ctypes.c_float * (1 << 14)).from_address(back.ptr))
    assert np.array_equal(x, y)
    assert len(list(tmp_path.iterdir())) == 1
    t.destroy()
    assert len(list(tmp_path.iterdir())) == 0


def direct_tree(G, cap=0):
    """FILE -> HBM siblings directly (the GDS edge, NEXT-4): no DRAM staging node."""
    t = nu.Tree()
    root = t.add_node(-1, nu.NU_FILE)
    for g in range(G):
        h = t.add_node(root, nu.NU_HBM, 0, cap)
        t.add_node(h, nu.NU_SMEM, 0, 227 * 1024, nu.NU_PROC_SM100)
    return t


@pytest.mark.parametrize("M,N,K,G,cap,panel,kind", [
    (512, 768, 1024, 1, 0, 256, "uniform"),
    (640, 900, 1500, 2, 0, 512, "int"),
    (1000, 1200, 3000, 1, 8_000_000, 1024, "int"),   # capacity -> several C blocks
    (300, 200, 130, 2, 0, 0, "int"),                  # row-major A: per-row reads
])
def test_file_direct_to_hbm(tmp_path, monkeypatch, M, N, K, G, cap, panel, kind):
    """The default FILE -> HBM transfer goes through the pinned bounce buffer
    (cuFile is opt-in, NORTHUP_CUFILE=1: its compat mode hung on this pool)."""
    monkeypatch.delenv("NORTHUP_CUFILE", raising=False)
    A = nugen.fill(M, K, 7, 1, kind)
    B = nugen.fill(K, N, 7, 2, kind)
    a_path, b_path, c_path = tmp_path / "A.bin", tmp_path / "B.bin", tmp_path / "C.bin"
    A.tofile(a_path)
    B.tofile(b_path)
    if panel:
        nu.file_tile_kpanels(str(a_path), str(tmp_path / "A_t.bin"), M, K, panel)
        a_path = tmp_path / "A_t.bin"
    t = direct_tree(G, cap)
    t.finalize()
    fa = t.open_file(0, str(a_path), 4 * M * K)
    fb = t.open_file(0, str(b_path), 4 * K * N)
    fc = t.open_file(0, str(c_path), 4 * M * N)
    st = t.gemm(fa, fb, fc, M, N, K, nu.make_opts(a_panel_k=panel))
    t.destroy()
    assert st["file_direct_mode"] == 2
    C = np.fromfile(c_path, dtype=np.float32).reshape(M, N)
    ref = oracle.gemm(A, B)
    if kind == "int":
        assert np.array_equal(C.astype(np.float64), ref)
    else:
        e, _ = oracle.normwise_err(C, ref, oracle.row_norms(A), oracle.col_norms(B))
        assert e <= 1e-5, e
    assert st["bytes_file_write"] == 4 * M * N


# ------------------------------------------------------------ I/O fault injection
# NORTHUP_IO_FAULT="<read|write>:<eio|enospc|short|eof>:<n>" (northup.h) makes the
# n-th pread / pwrite of the process fail; each case runs in its own process.
_FAULT_SCRIPT = r'''
import ctypes, json, sys
import numpy as np
sys.path.insert(0, {root!r})
import nugen, oracle
import paper_conf_ipps_chey19_b200 as nu
d = {d!r}
out = {{}}
M, N, K = 256, 192, 320
A = nugen.fill(M, K, 9, 1, "int"); B = nugen.fill(K, N, 9, 2, "int")
A.tofile(d + "/A.bin"); B.tofile(d + "/B.bin")
t = nu.Tree(); root = t.add_node(-1, nu.NU_FILE); st = t.add_node(root, nu.NU_HOST)
h = t.add_node(st, nu.NU_HBM, 0); t.add_node(h, nu.NU_SMEM, 0, 227 * 1024, nu.NU_PROC_SM100)
t.finalize()
fa = t.open_file(0, d + "/A.bin", 4 * M * K); fb = t.open_file(0, d + "/B.bin", 4 * K * N)
fc = t.open_file(0, d + "/C.bin", 4 * M * N)
try:
    t.gemm(fa, fb, fc, M, N, K, nu.make_opts(k_chunk=64))
    C = np.fromfile(d + "/C.bin", dtype=np.float32).reshape(M, N)
    out["rc"] = 0
    out["exact"] = bool(np.array_equal(C.astype(np.float64), oracle.gemm(A, B)))
except nu.NorthupError as e:
    out["rc"] = e.code
    out["msg"] = str(e)
out["errno"] = nu.last_io_errno()
t.destroy()
print(json.dumps(out))
'''


def _run_fault(tmp_path, spec):
    import json
    import os
    import subprocess
    import sys
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    env = dict(os.environ)
    if spec:
        env["NORTHUP_IO_FAULT"] = spec
    r = subprocess.run([sys.executable, "-c", _FAULT_SCRIPT.format(root=root, d=str(tmp_path))],
                       capture_output=True, text=True, timeout=300, env=env)
    assert r.returncode == 0, r.stderr[-2000:]
    return json.loads(r.stdout.strip().splitlines()[-1])


@pytest.mark.parametrize("spec,err", [("read:eio:3", 5), ("write:enospc:1", 28), ("read:eof:2", 0)])
def test_file_io_faults_fail_loudly(tmp_path, spec, err):
    """An I/O error on the FILE path ends northup_gemm with NU_EIO (no hang,
    Listing 4's file_read / file_write) and keeps the errno."""
    out = _run_fault(tmp_path, spec)
    assert out["rc"] == nu.NU_EIO and out["errno"] == err, out
    assert ("pread" in out["msg"]) == spec.startswith("read") and ("pwrite" in out["msg"]) == spec.startswith("write")


@pytest.mark.parametrize("spec", ["read:short:2", "write:short:1", ""])
def test_file_short_transfers_are_completed(tmp_path, spec):
    """pread / pwrite may move fewer bytes than asked: the library loops, so
    the result is still exact."""
    out = _run_fault(tmp_path, spec)
    assert out["rc"] == 0 and out["exact"], out


# -------------------------------------------- Listing 2 vs Listing 3
def _listing2(a_path, b_path, c_path, M, N, K, L0, L1, kc):
    """PAPER.md Listing 2, written out for this machine: the file (level 0) is
    cut into L0 x L0 chunks of C, each chunk's A rows / B columns are read into
    a DRAM buffer (level 1), cut into L1 x L1 sub-chunks, each copied to the
    GPU (level 2), computed there by the leaf kernel one K panel of `kc` at a
    time, copied back, and the DRAM result written to the result file."""
    import torch
    dev = torch.device("cuda:0")
    fa = np.memmap(a_path, dtype=np.float32, mode="r", shape=(M, K))
    fb = np.memmap(b_path, dtype=np.float32, mode="r", shape=(K, N))
    fc = np.memmap(c_path, dtype=np.float32, mode="w+", shape=(M, N))
    cut = lambda n, p: [(n * i // p, n * (i + 1) // p) for i in range(p)]
    for (i0, i1) in cut(M, L0):
        for (j0, j1) in cut(N, L0):
            buf_a = np.array(fa[i0:i1])                       # file_read -> DRAM
            buf_b = np.array(fb[:, j0:j1])
            result = np.empty((i1 - i0, j1 - j0), np.float32)
            for (m0, m1) in cut(i1 - i0, L1):
                for (n0, n1) in cut(j1 - j0, L1):
                    d_a = torch.from_numpy(buf_a[m0:m1]).to(dev)          # dCopyBlockH2D
                    d_b = torch.from_numpy(np.ascontiguousarray(buf_b[:, n0:n1])).to(dev)
                    d_c = torch.empty((m1 - m0, n1 - n0), device=dev)
                    for k0 in range(0, K, kc):                          # dLaunchComputation
                        k1 = min(K, k0 + kc)
                        nu.leaf_gemm(d_a[:, k0:k1], d_b[k0:k1], d_c, accumulate=k0 > 0)
                    result[m0:m1, n0:n1] = d_c.cpu().numpy()             # dCopyBlockD2H
            fc[i0:i1, j0:j1] = result                         # file_write
    fc.flush()
    del fc


@pytest.mark.parametrize("M,N,K,kc,cap", [
    (1000, 1200, 3000, 1024, 8_000_000),     # several C blocks, ragged last panel
    (777, 515, 2049, 512, 0),
])
def test_listing2_equals_recursive_engine(tmp_path, M, N, K, kc, cap):
    """SURVEY §4 T4 / P:224: the hard-coded two-level loop of Listing 2 and the
    recursive engine of Listing 3 (northup_gemm over FILE -> HOST -> HBM ->
    SMEM) give bitwise identical C on uniform inputs when both run the leaf
    over the same K-panel sequence - the recursion only changes where data
    lives, never the arithmetic."""
    A = nugen.fill(M, K, 31, 1)
    B = nugen.fill(K, N, 31, 2)
    a_path, b_path = tmp_path / "A.bin", tmp_path / "B.bin"
    A.tofile(a_path)
    B.tofile(b_path)
    _listing2(str(a_path), str(b_path), str(tmp_path / "C2.bin"), M, N, K, 2, 2, kc)
    C2 = np.fromfile(tmp_path / "C2.bin", dtype=np.float32).reshape(M, N)
    t = file_tree(1, cap)
    t.finalize()
    st = t.gemm(t.open_file(0, str(a_path), 4 * M * K), t.open_file(0, str(b_path), 4 * K * N),
                t.open_file(0, str(tmp_path / "C3.bin"), 4 * M * N), M, N, K, nu.make_opts(k_chunk=kc))
    t.destroy()
    C3 = np.fromfile(tmp_path / "C3.bin", dtype=np.float32).reshape(M, N)
    e, _ = oracle.normwise_err(C3, oracle.gemm(A, B), oracle.row_norms(A), oracle.col_norms(B))
    assert e <= 1e-5, e
    assert np.array_equal(C2, C3)
    if cap:
        assert st["leaf_launches"] > 3
