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
