"""Small runs of the paths changed late in round 1, for compute-sanitizer (memcheck /
synccheck): the product leaf on ragged shapes, a HOST -> 2 x HBM tree with shared
staging (virtual siblings), the FILE -> HBM edge through the pipelined bounce, a FILE root
with DRAM staging (two I/O threads), and the HotSpot tree with split first/last blocks."""
import os, sys, tempfile
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import nugen
import paper_conf_ipps_chey19_b200 as nu

dev = torch.device("cuda:0")
for (M, N, K) in [(300, 300, 132), (257, 520, 2100), (130, 72, 40)]:
    A = torch.from_numpy(nugen.fill(M, K, 1, 1)).to(dev)
    B = torch.from_numpy(nugen.fill(K, N, 1, 2)).to(dev)
    C = torch.empty((M, N), device=dev)
    nu.leaf_gemm(A, B, C, k_chunk=512)
torch.cuda.synchronize()


def host_gemm(G, M, N, K, cap=0):
    t, _ = nu.host_tree(G, cap, devices=[0] * G)
    t.finalize()
    a, b, c = t.alloc(4 * M * K, 0), t.alloc(4 * K * N, 0), t.alloc(4 * M * N, 0)
    st = t.gemm(a, b, c, M, N, K, nu.make_opts(k_chunk=256))
    t.destroy()
    return st


st = host_gemm(2, 640, 512, 1024)
assert st["shared_staging"] == 1
d = tempfile.mkdtemp()
M, N, K = 900, 700, 700
nugen.fill(M, K, 2, 1).tofile(f"{d}/A.bin")
nugen.fill(K, N, 2, 2).tofile(f"{d}/B.bin")
for staging in (False, True):
    t = nu.Tree()
    root = t.add_node(-1, nu.NU_FILE)
    par = t.add_node(root, nu.NU_HOST, -1, 0) if staging else root
    h = t.add_node(par, nu.NU_HBM, 0, 6_000_000)
    t.add_node(h, nu.NU_SMEM, 0, 227 * 1024, nu.NU_PROC_SM100)
    t.finalize()
    fa, fb = t.open_file(0, f"{d}/A.bin", 4 * M * K), t.open_file(0, f"{d}/B.bin", 4 * K * N)
    fc = t.open_file(0, f"{d}/C{int(staging)}.bin", 4 * M * N)
    t.gemm(fa, fb, fc, M, N, K)
    t.destroy()
R, C_, it = 600, 520, 9
t, _ = nu.host_tree(1)
t.finalize()
Tb, Pb, Ob = t.alloc(4 * R * C_, 0), t.alloc(4 * R * C_, 0), t.alloc(4 * R * C_, 0)
t.hotspot(Tb, Pb, Ob, R, C_, it, nu.hotspot_opts(block=300, halo=4, leaf_iters=4))
t.destroy()
torch.cuda.synchronize()
print("sanitize3 ok")
