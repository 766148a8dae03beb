"""cfg3 out-of-core time with (GRAPH=1) or without CUDA-graph replay of the op lists.
Prints one JSON line (best of 4 calls after 2 warm-ups)."""
import ctypes, json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np
import nugen
import paper_conf_ipps_chey19_b200 as nu
M = N = K = 32768
t, _ = nu.host_tree(1, 8 << 30)
t.finalize()
A, B, C = t.alloc(4 * M * K, 0), t.alloc(4 * K * N, 0), t.alloc(4 * M * N, 0)
v = lambda b, r, c: np.ctypeslib.as_array((ctypes.c_float * (r * c)).from_address(b.ptr)).reshape(r, c)
nugen.fill(M, K, 3, nugen.MAT_A, out=v(A, M, K))
nugen.fill(K, N, 3, nugen.MAT_B, out=v(B, K, N))
o = nu.make_opts(k_chunk=2048, graph=os.environ.get("GRAPH") == "1")
for _ in range(2):
    st = t.gemm(A, B, C, M, N, K, o)
ms = []
for _ in range(4):
    t0 = time.perf_counter()
    st = t.gemm(A, B, C, M, N, K, o)
    ms.append((time.perf_counter() - t0) * 1e3)
print(json.dumps({"graph": os.environ.get("GRAPH") == "1", "graph_replayed": st.get("graph_replayed"), "tail_k": st["tail_k"], "strips": st["strips"], "ms": round(min(ms), 2),
                  "tflops": round(2.0 * M * N * K / min(ms) / 1e9, 1)}))
