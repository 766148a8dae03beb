"""Debug harness for the leaf kernel: variants + smem stage dump."""
import ctypes, sys, os
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import nugen, oracle
import paper_conf_ipps_chey19_b200 as nu

L = nu.lib()
f = L.northup_debug_leaf_gemm
f.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
              ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int,
              ctypes.c_int64, ctypes.c_int, ctypes.c_int, ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p]
f.restype = ctypes.c_int
dev = torch.device("cuda:0")

def unswz(buf, rows, rowbytes=128):
    # 128B swizzle: 16-byte chunk j of row r sits at chunk j ^ (r % 8)
    b = buf.view(np.uint8).reshape(rows, rowbytes)
    out = np.empty_like(b)
    for r in range(rows):
        for j in range(rowbytes // 16):
            jj = j ^ (r % 8)
            out[r, j*16:(j+1)*16] = b[r, jj*16:(jj+1)*16]
    return out.view(np.float32)

def unswz32(buf, rows):
    # 128B rows, 32-byte granules XOR (row % 4)
    b = buf.view(np.uint8).reshape(rows, 128)
    out = np.empty_like(b)
    for r in range(rows):
        for j in range(4):
            jj = j ^ (r % 4)
            out[r, j*32:(j+1)*32] = b[r, jj*32:(jj+1)*32]
    return out.view(np.float32)

def run(M, N, K, kind, npass, bk, variant=1):
    A = nugen.fill(M, K, 11, 1, kind); B = nugen.fill(K, N, 11, 2, kind)
    Ad = torch.from_numpy(A).to(dev)
    Bd = torch.from_numpy(np.ascontiguousarray(B.T) if bk else B).to(dev)
    Cd = torch.full((M, N), float('nan'), device=dev)
    dbg = torch.zeros(96 * 1024 // 4, device=dev)
    rc = f(Ad.data_ptr(), K, Bd.data_ptr(), Bd.stride(0), Cd.data_ptr(), N, M, N, K, 0, 0, npass, bk,
           dbg.data_ptr() if variant == 1 else None, variant, None)
    if rc: print("rc", rc, nu.last_error()); return
    torch.cuda.synchronize()
    C = Cd.cpu().numpy(); ref = oracle.gemm(A, B)
    err = np.abs(C - ref).max()
    print(f"M{M} N{N} K{K} {kind} npass={npass} b_kmajor={bk} variant={variant}: max abs err {err:.3e}; C[0,:4]={C[0,:4]} ref={ref[0,:4]}")
    if npass == 1 and kind == "uniform":
        tr = lambda x: (x.view(np.uint32) & np.uint32(0xFFFFE000)).view(np.float32)
        rn = lambda x: ((x.view(np.uint32) + np.uint32(0x1000)) & np.uint32(0xFFFFE000)).view(np.float32)
        ct = tr(A).astype(np.float64) @ tr(B).astype(np.float64)
        cr = rn(A).astype(np.float64) @ rn(B).astype(np.float64)
        print(f"  HW operand rounding probe: |C-trunc| {np.abs(C-ct).max():.3e}  |C-rna| {np.abs(C-cr).max():.3e}")
    if variant != 1: return C, ref
    d = dbg.cpu().numpy()
    a_raw = unswz(d[:128*32].copy(), 128)
    print("  A stage (hi) == trunc(A):", np.array_equal(a_raw[:M, :min(K,32)], (A.view(np.uint32) & 0xFFFFE000).view(np.float32)[:, :32][:M, :min(K,32)]))
    boff = 128*32
    if bk:
        b_raw = unswz(d[boff:boff+256*32].copy(), 256)
        print("  B stage (K-major) == B^T:", np.array_equal(b_raw[:N, :min(K,32)], np.ascontiguousarray(B.T)[:, :32]))
    else:
        ok = True
        for c in range(8):
            chunk = unswz32(d[boff + c*1024: boff + (c+1)*1024].copy(), 32)
            ok &= np.array_equal(chunk[:min(K,32)], B[:32, c*32:(c+1)*32])
        print("  B stage (MN-major chunks) == B:", ok)
    return C, ref

for args in [(128, 256, 32, "uniform", 1, 0), (128, 256, 64, "uniform", 1, 0),
             (256, 256, 32, "int", 3, 0, 2), (256, 256, 32, "int", 1, 0, 2), (512, 512, 256, "int", 3, 0, 2),
             (300, 700, 333, "int", 3, 0, 2), (1024, 1024, 2048, "uniform", 3, 0, 2), (1024, 1024, 2048, "uniform", 3, 0, 1)]:
    try:
        run(*args)
    except Exception as e:
        print("EXC", args, e)
