"""One multi-process sibling for tests/test_gpu_peer.py (run as a script, one
process per sibling): builds the shared tree, runs only its HBM node
(northup_tree_set_local), exchanges CUDA IPC blobs with the other processes
through files in a rendezvous directory, and saves its C region."""
import ctypes
import os
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import numpy as np  # noqa: E402

import nugen  # noqa: E402
import paper_conf_ipps_chey19_b200 as nu  # noqa: E402


def wait_for(paths, timeout=120):
    t0 = time.time()
    while not all(os.path.exists(p) for p in paths):
        if time.time() - t0 > timeout:
            raise TimeoutError(f"rendezvous timed out waiting for {paths}")
        time.sleep(0.01)


def main():
    d, rank, G, M, N, K, kc, shared, kind, reps = sys.argv[1:11]
    rank, G, M, N, K, kc, shared, reps = map(int, (rank, G, M, N, K, kc, shared, reps))
    t, hbm = nu.host_tree(G, devices=[0] * G)        # all siblings on GPU 0 (1-GPU pool)
    t.set_local(hbm[rank])
    t.finalize()
    r0, r1, c0, c1 = nu.partition_region(G, M, N, K, rank)
    m, n = r1 - r0, c1 - c0
    A, B, C = t.alloc(4 * m * K, 0), t.alloc(4 * K * n, 0), t.alloc(4 * m * n, 0)
    view = lambda b, r, c: np.ctypeslib.as_array((ctypes.c_float * (r * c)).from_address(b.ptr)).reshape(r, c)
    a, b, c = view(A, m, K), view(B, K, n), view(C, m, n)
    nugen.fill(m, K, 5, nugen.MAT_A, kind, out=a, i0=r0, ncols=K)
    nugen.fill(K, n, 5, nugen.MAT_B, kind, out=b, j0=c0, ncols=N)
    o = nu.make_opts(k_chunk=kc, shared_staging=shared)
    if shared >= 0:
        blob = t.peer_export(M, N, K, o)
        with open(os.path.join(d, f"blob{rank}.tmp"), "wb") as f:
            f.write(blob)
        os.replace(os.path.join(d, f"blob{rank}.tmp"), os.path.join(d, f"blob{rank}"))
        wait_for([os.path.join(d, f"blob{w}") for w in range(G)])
        for w in range(G):
            if w != rank:
                t.peer_import(w, open(os.path.join(d, f"blob{w}"), "rb").read())
    if os.environ.get("PEER_SKIP_GEMM") == str(rank):
        # a sibling that never runs its part: the others must fail, not hang
        wait_for([os.path.join(d, f"err{w}") for w in range(G) if w != rank], timeout=240)
        open(os.path.join(d, f"done{rank}"), "w").close()
        return
    outs = []
    for _ in range(reps):
        c[...] = np.nan
        try:
            st = t.gemm(A, B, C, M, N, K, o)
        except nu.NorthupError as ex:
            open(os.path.join(d, f"err{rank}"), "w").write(str(ex))
            print("NorthupError:", ex, flush=True)
            os._exit(3)
        outs.append(c.copy())
    np.save(os.path.join(d, f"c{rank}.npy"), np.stack(outs))
    with open(os.path.join(d, f"st{rank}.txt"), "w") as f:
        f.write(f"{st['shared_staging']} {st['bytes_p2p']} {st['bytes_h2d']}\n")
    open(os.path.join(d, f"done{rank}"), "w").close()
    wait_for([os.path.join(d, f"done{w}") for w in range(G)])   # peers may map our arena
    t.destroy()


if __name__ == "__main__":
    main()
