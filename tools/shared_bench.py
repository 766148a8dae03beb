"""NEXT-1 on one B200: G virtual siblings (HBM nodes aliasing GPU 0) run an
out-of-core GEMM from pinned host memory with and without shared staging.
Sharing cuts the PCIe bytes from 4K(M Pc + N Pr) to 4K(M + N); the pulls are
device-local copies here (NVLink P2P between real siblings).  Also probes the
box's PCIe H2D / D2H bandwidth alone and concurrently (the roofline's staging
term).  Usage: python tools/shared_bench.py [M N K G cap_gib] ..."""
import ctypes, json, os, sys, time
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import numpy as np, torch
import nugen
import paper_conf_ipps_chey19_b200 as nu

GiB = 1 << 30


def pcie_probe(nbytes=2 * GiB, reps=3):
    h = torch.empty(nbytes // 4, dtype=torch.float32).pin_memory()
    h2 = torch.empty(nbytes // 4, dtype=torch.float32).pin_memory()
    d = torch.empty(nbytes // 4, dtype=torch.float32, device="cuda")
    d2 = torch.empty(nbytes // 4, dtype=torch.float32, device="cuda")
    s1, s2 = torch.cuda.Stream(), torch.cuda.Stream()
    out = {}
    for name, fn in [("h2d", lambda: d.copy_(h, non_blocking=True)),
                     ("d2h", lambda: h2.copy_(d2, non_blocking=True))]:
        fn(); torch.cuda.synchronize()
        t0 = time.perf_counter()
        for _ in range(reps): fn()
        torch.cuda.synchronize()
        out[name + "_gbs"] = reps * nbytes / (time.perf_counter() - t0) / 1e9
    torch.cuda.synchronize()
    t0 = time.perf_counter()
    for _ in range(reps):
        with torch.cuda.stream(s1): d.copy_(h, non_blocking=True)
        with torch.cuda.stream(s2): h2.copy_(d2, non_blocking=True)
    torch.cuda.synchronize()
    out["duplex_each_gbs"] = reps * nbytes / (time.perf_counter() - t0) / 1e9
    return out


def run(M, N, K, G, cap, steps=2):
    t, _ = nu.host_tree(G, cap, devices=[0] * G)
    t.finalize()
    A, B, C = t.alloc(4 * M * K, 0), t.alloc(4 * K * N, 0), t.alloc(4 * M * N, 0)
    arr = lambda b, r, c: np.ctypeslib.as_array((ctypes.c_float * (r * c)).from_address(b.ptr)).reshape(r, c)
    nugen.fill(M, K, 3, 1, out=arr(A, M, K))
    nugen.fill(K, N, 3, 2, out=arr(B, K, N))
    res = {"M": M, "N": N, "K": K, "G": G, "cap_gib": cap / GiB, "grid": nu.partition(G, M, N)}
    ref = None
    for sh in (-1, 0):
        o = nu.make_opts(shared_staging=sh)
        t.gemm(A, B, C, M, N, K, o)                    # warm-up (arena allocation)
        ms = []
        for _ in range(steps):
            torch.cuda.synchronize()
            t0 = time.perf_counter()
            st = t.gemm(A, B, C, M, N, K, o)
            ms.append((time.perf_counter() - t0) * 1e3)
        c = arr(C, M, N).copy()
        if ref is None:
            ref = c
        tim = t.gemm(A, B, C, M, N, K, nu.make_opts(shared_staging=sh, collect_timing=True))
        key = "shared" if sh == 0 else "unshared"
        res[key] = {"ms": min(ms), "tflops": 2.0 * M * N * K / (min(ms) * 1e-3) / 1e12,
                    "h2d_gib": st["bytes_h2d"] / GiB, "p2p_gib": st["bytes_p2p"] / GiB,
                    "d2h_gib": st["bytes_d2h"] / GiB, "shared_staging": st["shared_staging"],
                    "tail_k": st["tail_k"], "blocks": [st["bm"], st["bn"], st["bk"]],
                    "busy_ms_sum_over_siblings": {"h2d": tim["t_h2d_ms"], "compute": tim["t_compute_ms"],
                                                  "d2h": tim["t_d2h_ms"], "p2p": tim["t_p2p_ms"]},
                    "h2d_gbs": st["bytes_h2d"] / max(tim["t_h2d_ms"], 1e-9) / 1e6}
    res["bitwise_shared_vs_unshared"] = bool(np.array_equal(ref, c))
    t.destroy()
    return res


if __name__ == "__main__":
    cases = [(32768, 32768, 32768, 4, 8 * GiB), (32768, 32768, 32768, 2, 8 * GiB),
             (65536, 16384, 8192, 8, 8 * GiB)]
    if len(sys.argv) > 1:
        v = list(map(int, sys.argv[1:]))
        cases = [(v[i], v[i + 1], v[i + 2], v[i + 3], v[i + 4] * GiB) for i in range(0, len(v), 5)]
    out = {"pcie": pcie_probe(), "cases": []}
    print(json.dumps(out["pcie"]), flush=True)
    for c in cases:
        r = run(*c)
        print(json.dumps(r), flush=True)
        out["cases"].append(r)
    os.makedirs("gpurun_out", exist_ok=True)
    with open("gpurun_out/shared_bench.json", "w") as f:
        json.dump(out, f, indent=1)
