#!/usr/bin/env python
"""Benchmark of the Northup out-of-core recursive GEMM on B200 (BASELINE.json
metric: "out-of-core GEMM TFLOP/s at 1/2/4/8 B200; % slowdown vs in-HBM;
roofline frac").

One step = one northup_gemm call = one pass of the whole hot path:
  value  : the out-of-core GEMM (the metric) through the C ABI from pinned
           HOST buffers (HOST -> HBM (8 GiB cap) -> SMEM/TMEM), every H2D/D2H
           inside the step; CUDA events bracketing the synchronous calls;
  e2e    : the same calls timed by the host clock (planning and issue included);
  in_hbm : the same GEMM with A, B, C resident in HBM (single-node HBM tree,
           CS4 — the paper's in-memory baseline).
  slowdown = t_value / t_in_hbm - 1.

N = 1 runs BASELINE configs[2] (cfg3: 32768^3, 8 GiB HBM cap).  Under torchrun
(N > 1) every rank runs its C region of configs[3] (cfg4: 65536 x 65536 x
32768, pinned-host root) — disjoint C subtrees, no data-path collective.

`--impl reference` times the fp64 CPU oracle (the only reference this paper
has) on a bounded sample of the same workload, on the host cores.
"""
from __future__ import annotations

import argparse
import ctypes
import json
import os
import statistics
import subprocess
import sys
import threading
import time

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

GiB = 1 << 30
METRIC = "out-of-core GEMM TFLOP/s at 1/2/4/8 B200; % slowdown vs in-HBM; roofline frac"
CONFIGS = {
    "cfg1": dict(M=256, N=256, K=256, cap=0, block=(64, 64, 64),
                 desc="256x256x256 fp32, host DRAM -> 1 GPU leaf, 64x64 blocks"),
    "cfg2": dict(M=8192, N=8192, K=8192, cap=0, block=None,
                 desc="8192^3 fp32 (in-HBM reference point)"),
    "cfg3": dict(M=32768, N=32768, K=32768, cap=8 * GiB, block=None,
                 desc="32768^3 fp32, pinned host -> HBM (8 GiB cap) -> SMEM/TMEM, 1 GPU"),
    "cfg4": dict(M=65536, N=65536, K=32768, cap=8 * GiB, block=None,
                 desc="65536x65536x32768 fp32, pinned-host root (no NVMe on the box), C subtrees over G GPUs"),
    "cfg5": dict(M=1048576, N=4096, K=4096, cap=8 * GiB, block=None,
                 desc="tall-skinny 1048576x4096x4096 fp32, A streamed from host"),
}
HOTSPOT = dict(R=32768, C=32768, iters=256, cap=8 * GiB,
               desc="HotSpot-2D 32768^2 fp32 grid (P:349 32k inputs) x 256 iterations, pinned host -> "
                    "HBM (8 GiB cap) -> SMEM, 1 GPU (S§8(f) NEXT-3)")
SCHEDULES = {"auto": 0, "s1": 1, "s2": 2, "queue": 3, "s2b": 4}
HS_FLOPS_PER_UPDATE = 14                 # flops of one cell update as the formula states (5 mul + 9 add/sub)
FP32_LANES_PER_SM, N_SMS = 128, 148      # B200: 4 SMSPs x 32 fp32 lanes; 148 SMs


def log(*a):
    print(*a, file=sys.stderr, flush=True)


# ------------------------------------------------------------------ clocks
class ClockSampler:
    """nvidia-smi clocks/throttle reasons sampled during the timed region."""

    FIELDS = ("index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active,"
              "clocks_event_reasons.hw_slowdown,clocks_event_reasons.hw_thermal_slowdown,"
              "clocks_event_reasons.sw_thermal_slowdown,clocks_event_reasons.sw_power_cap")

    def __init__(self, gpu: int):
        self.gpu = gpu
        self.rows = []
        self.proc = None

    def __enter__(self):
        try:
            self.proc = subprocess.Popen(
                ["nvidia-smi", "-i", str(self.gpu), f"--query-gpu={self.FIELDS}",
                 "--format=csv,noheader,nounits", "-lms", "200"],
                stdout=subprocess.PIPE, stderr=subprocess.DEVNULL, text=True)
            self.th = threading.Thread(target=self._read, daemon=True)
            self.th.start()
        except FileNotFoundError:
            self.proc = None
        return self

    def _read(self):
        for line in self.proc.stdout:
            parts = [p.strip() for p in line.split(",")]
            if len(parts) >= 9:
                self.rows.append(parts)

    def __exit__(self, *exc):
        if self.proc:
            self.proc.terminate()
            try:
                self.proc.wait(timeout=5)
            except subprocess.TimeoutExpired:
                self.proc.kill()

    def summary(self) -> dict:
        if not self.rows:
            return {"sm_mhz": None, "sm_max_mhz": None, "reasons": ["unsampled"]}
        def num(x):
            try:
                return float(x)
            except ValueError:
                return None
        sm = [num(r[1]) for r in self.rows if num(r[1])]
        mx = [num(r[2]) for r in self.rows if num(r[2])]
        pw = [num(r[3]) for r in self.rows if num(r[3])]
        names = ["hw_slowdown", "hw_thermal_slowdown", "sw_thermal_slowdown", "sw_power_cap"]
        reasons = sorted({names[i] for r in self.rows for i in range(4)
                          if r[5 + i].lower().startswith("active")})
        loaded = sorted(sm)[len(sm) // 2:] if sm else []
        return {"sm_mhz": statistics.median(loaded) if loaded else None,
                "sm_max_mhz": max(mx) if mx else None,
                "power_w_max": max(pw) if pw else None,
                "samples": len(self.rows), "reasons": reasons}


# ------------------------------------------------------------------ peaks
def measured_peaks() -> dict:
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        return {"bf16_burst": d["bf16_tflops"], "bf16_sustained": d.get("bf16_tflops_sustained",
                d["bf16_tflops"]), "hbm_gbs": d["hbm_gbs"], "source": "measured"}
    return {"bf16_burst": 1590.0, "bf16_sustained": 1400.0, "hbm_gbs": 6650.0, "source": "fallback"}


def measure_pcie(dev, nbytes: int = 1 << 30, reps: int = 5) -> dict:
    """Pinned host <-> HBM copy bandwidth on this GPU's link (GB/s): H2D alone,
    D2H alone and both directions at once (the out-of-core schedule runs both);
    best of `reps`, CUDA events on the copy streams."""
    import torch
    h_in = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    h_out = torch.empty(nbytes, dtype=torch.uint8, pin_memory=True)
    d_in = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    d_out = torch.empty(nbytes, dtype=torch.uint8, device=dev)
    s1, s2 = torch.cuda.Stream(dev), torch.cuda.Stream(dev)

    def run(h2d: bool, d2h: bool) -> tuple:
        best = (0.0, 0.0)
        for _ in range(reps):
            torch.cuda.synchronize(dev)
            ev = [torch.cuda.Event(enable_timing=True) for _ in range(4)]
            if h2d:
                ev[0].record(s1)
                with torch.cuda.stream(s1):
                    d_in.copy_(h_in, non_blocking=True)
                ev[1].record(s1)
            if d2h:
                ev[2].record(s2)
                with torch.cuda.stream(s2):
                    h_out.copy_(d_out, non_blocking=True)
                ev[3].record(s2)
            torch.cuda.synchronize(dev)
            bw = (nbytes / (ev[0].elapsed_time(ev[1]) * 1e6) if h2d else 0.0,
                  nbytes / (ev[2].elapsed_time(ev[3]) * 1e6) if d2h else 0.0)
            best = (max(best[0], bw[0]), max(best[1], bw[1]))
        return best

    h2d, _ = run(True, False)
    _, d2h = run(False, True)
    bh, bd = run(True, True)
    del h_in, h_out, d_in, d_out
    return {"h2d_gbs": round(h2d, 2), "d2h_gbs": round(d2h, 2), "bidir_h2d_gbs": round(bh, 2),
            "bidir_d2h_gbs": round(bd, 2), "link": "PCIe Gen5 x16 (64 GB/s per direction raw)",
            "how": f"pinned {nbytes >> 20} MiB copies, best of {reps}, CUDA events"}


def ooc_roofline(flops: float, bytes_h2d: int, bytes_d2h: int, p_eff: float, pcie: dict) -> dict:
    """S§8(d) per-GPU roofline R = min(P_eff, BW_h2d * I_h2d, BW_d2h * I_d2h) at the
    planner's block size: I_e = useful flops / bytes the schedule moves over edge e,
    BW_e = the link bandwidth measured with both directions active."""
    terms = {"tensor": p_eff}
    if bytes_h2d:
        terms["pcie_h2d"] = pcie["bidir_h2d_gbs"] * 1e9 * flops / bytes_h2d / 1e12
    if bytes_d2h:
        terms["pcie_d2h"] = pcie["bidir_d2h_gbs"] * 1e9 * flops / bytes_d2h / 1e12
    bound = min(terms, key=terms.get)
    return {"bound": bound, "peak": round(terms[bound], 3), "unit": "TFLOP/s",
            "terms": {k: round(v, 3) for k, v in terms.items()},
            "intensity_flop_per_byte": {"h2d": round(flops / bytes_h2d, 1) if bytes_h2d else None,
                                        "d2h": round(flops / bytes_d2h, 1) if bytes_d2h else None}}


def host_array(ptr: int, rows: int, cols: int):
    import numpy as np
    n = rows * cols
    return np.ctypeslib.as_array((ctypes.c_float * n).from_address(ptr)).reshape(rows, cols)


# ------------------------------------------------------------- CPU oracle leg
def cpu_baseline(cfg: dict, a_host, b_host, c_gpu, budget_s: float) -> dict:
    """The fp64 oracle timed on a bounded sample (full rows of C) on the host
    cores; also reports the normwise error of the GPU's C on those rows."""
    import numpy as np
    import oracle
    M, N, K = cfg["M"], cfg["N"], cfg["K"]
    cores = len(os.sched_getaffinity(0))
    oracle.set_threads(cores)
    rng = np.random.default_rng(12345)
    rows = np.sort(rng.choice(M, size=min(M, cores), replace=False))
    t0 = time.perf_counter()
    ref = oracle.gemm_rows(a_host, b_host, rows)
    dt = time.perf_counter() - t0
    done = [(rows, ref)]
    nrows, elapsed = len(rows), dt
    # grow the sample up to the time budget (whole multiples of `cores` rows)
    if dt > 0 and dt < budget_s / 2:
        reps = max(1, int((budget_s - dt) / dt))
        more = np.sort(rng.choice(M, size=min(M, reps * cores), replace=False))
        t0 = time.perf_counter()
        ref2 = oracle.gemm_rows(a_host, b_host, more)
        elapsed += time.perf_counter() - t0
        nrows += len(more)
        done.append((more, ref2))
    flops = 2.0 * nrows * N * K
    # the same oracle on one core (a single row of C)
    oracle.set_threads(1)
    t0 = time.perf_counter()
    oracle.gemm_rows(a_host, b_host, rows[:1])
    one = 2.0 * N * K / (time.perf_counter() - t0) / 1e12
    oracle.set_threads(cores)
    out = {"value": flops / elapsed / 1e12, "unit": "TFLOP/s", "cores": cores, "kind": "oracle",
           "sample": f"{nrows} full rows of C ({nrows}x{N}x{K} fp64 triple loop), {elapsed:.1f} s",
           "seconds": elapsed, "single_core_value": one, **cpu_facts()}
    if c_gpu is not None:
        cn = oracle.col_norms(b_host)
        worst = 0.0
        for rws, rf in done:
            a_s = np.ascontiguousarray(a_host[rws])
            e, _ = oracle.normwise_err(np.ascontiguousarray(c_gpu[rws]), rf, oracle.row_norms(a_s), cn)
            worst = max(worst, e)
        out["gpu_normwise_err_on_sample"] = worst
        out["gpu_parity_ok"] = bool(worst <= 1e-5)
    return out


# -------------------------------------------------------------- host facts
def cpu_facts() -> dict:
    model = None
    try:
        with open("/proc/cpuinfo") as f:
            for line in f:
                if line.startswith("model name"):
                    model = line.split(":", 1)[1].strip()
                    break
    except OSError:
        pass
    nodes = [d for d in os.listdir("/sys/devices/system/node") if d.startswith("node") and d[4:].isdigit()] \
        if os.path.isdir("/sys/devices/system/node") else []
    return {"cpu_model": model, "numa_nodes": len(nodes) or 1, "logical_cpus": os.cpu_count()}


def _cpulist(text: str) -> set:
    cpus = set()
    for part in text.strip().split(","):
        if not part:
            continue
        if "-" in part:
            a, b = part.split("-")
            cpus.update(range(int(a), int(b) + 1))
        else:
            cpus.add(int(part))
    return cpus


def bind_to_gpu_numa(dev_index: int) -> dict:
    """Bind this process (and the threads it starts: the library's per-GPU
    workers, the generator's OpenMP threads) to the NUMA node of its GPU, so
    the pinned root strips are first-touched next to the GPU's PCIe link
    (SURVEY §7 H5).  Returns what was done; a no-op on one-node hosts."""
    import torch
    info = {"gpu": dev_index, "numa_node": None, "cpus": None, "bound": False}
    try:
        p = torch.cuda.get_device_properties(dev_index)
        bus = "%04x:%02x:%02x.0" % (p.pci_domain_id, p.pci_bus_id, p.pci_device_id)
        with open(f"/sys/bus/pci/devices/{bus}/numa_node") as f:
            node = int(f.read().strip())
        info["numa_node"] = node
        if node < 0:
            return info
        with open(f"/sys/devices/system/node/node{node}/cpulist") as f:
            cpus = _cpulist(f.read()) & os.sched_getaffinity(0)
        if cpus and len(cpus) < len(os.sched_getaffinity(0)):
            os.sched_setaffinity(0, cpus)
            info.update(cpus=len(cpus), bound=True)
    except (OSError, AttributeError, ValueError) as ex:
        info["error"] = repr(ex)
    return info


def kernel_launches() -> int:
    import paper_conf_ipps_chey19_b200 as nu
    f = nu.lib().northup_debug_kernel_launches
    f.restype = ctypes.c_longlong
    return int(f())


def leaf_kernel_ms(A, B, C, kc: int, stream, reps: int = 2) -> list:
    """Device time of each GEMM kernel launch of the leaf (CUDA events recorded
    by the library around the kernel, on `stream`): the dominant kernel."""
    import torch
    import paper_conf_ipps_chey19_b200 as nu
    f = nu.lib().northup_debug_leaf_gemm_events
    f.argtypes = [ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p, ctypes.c_int64, ctypes.c_void_p,
                  ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64, ctypes.c_int64,
                  ctypes.c_void_p, ctypes.c_void_p, ctypes.c_int, ctypes.c_void_p]
    M, K = A.shape
    N = B.shape[1]
    nev = 2 * (-(-K // kc)) * (-(-N // 32768))
    out = []
    for _ in range(reps):
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(nev)]
        for e in evs:
            e.record(stream)            # creates the events on this device
        handles = (ctypes.c_void_p * nev)(*[e.cuda_event for e in evs])
        used = ctypes.c_int(0)
        nu.check(f(A.data_ptr(), A.stride(0), B.data_ptr(), B.stride(0), C.data_ptr(), C.stride(0), M, N, K, kc,
                   stream.cuda_stream, handles, nev, ctypes.byref(used)))
        torch.cuda.synchronize()
        out += [evs[i].elapsed_time(evs[i + 1]) for i in range(0, used.value, 2)]
    return out


# -------------------------------------------------------------------- ours
def run_ours(args, rank: int, world: int, local_rank: int):
    import numpy as np
    import torch
    import nugen
    import paper_conf_ipps_chey19_b200 as nu

    dist = None
    if world > 1:
        import torch.distributed as dist
    dev = torch.device("cuda", local_rank)
    torch.cuda.set_device(dev)
    all_cpus = os.sched_getaffinity(0)
    numa = bind_to_gpu_numa(local_rank) if not args.no_numa_bind else {"bound": False, "disabled": True}
    name = args.config or ("cfg3" if world == 1 else "cfg4")
    cfg = dict(CONFIGS[name])
    if args.quick:
        cfg.update(M=cfg["M"] // 4, N=cfg["N"] // 4, K=cfg["K"] // 4, cap=cfg["cap"] // 4)
    M, N, K = cfg["M"], cfg["N"], cfg["K"]
    r0, r1, c0, c1 = nu.partition_region(world, M, N, K, rank) if world > 1 else (0, M, 0, N)
    m, n = r1 - r0, c1 - c0
    seed = int(name[-1])
    kc = args.k_chunk
    if cfg["block"]:
        # a fixed block (cfg1's 64 x 64 x 64) fixes the K-panel sequence: the in-HBM
        # reference runs the same panels, so the two stay bitwise comparable
        kc = cfg["block"][2]

    # --- the out-of-core tree: HOST root -> HBM (cap) -> SMEM/TMEM leaf.  N > 1:
    # the same tree on every rank (one HBM sibling per rank); this rank runs
    # only its own sibling (multi-process siblings, northup_tree_set_local).
    if world > 1:
        devs = [(i % args.device_mod) if args.device_mod > 0 else i for i in range(world)]
        t, hbm = nu.host_tree(world, cfg["cap"], devices=devs)
        t.set_local(hbm[rank])
    else:
        t, hbm = nu.host_tree(1, cfg["cap"], devices=[local_rank])
    if cfg["block"]:
        t.set_block(0, *cfg["block"])
    t.finalize()
    tg = time.perf_counter()
    Ab, Bb, Cb = t.alloc(4 * m * K, 0), t.alloc(4 * K * n, 0), t.alloc(4 * m * n, 0)
    a = host_array(Ab.ptr, m, K)
    b = host_array(Bb.ptr, K, n)
    c = host_array(Cb.ptr, m, n)
    nugen.fill(m, K, seed, nugen.MAT_A, "uniform", out=a, i0=r0, ncols=K)
    nugen.fill(K, n, seed, nugen.MAT_B, "uniform", out=b, j0=c0, ncols=N)
    log(f"[rank {rank}] {name} region {m}x{n}x{K}: inputs generated in pinned host memory "
        f"in {time.perf_counter() - tg:.1f} s (NUMA {numa})")

    # --- the in-HBM tree (CS4): the same GEMM with A, B, C resident in HBM
    th = nu.hbm_tree(local_rank)
    th.finalize()
    Ad = torch.from_numpy(a).to(dev)
    Bd = torch.from_numpy(b).to(dev)
    Cd = torch.empty((m, n), dtype=torch.float32, device=dev)
    hA = th.wrap_device(0, Ad.data_ptr(), Ad.numel() * 4)
    hB = th.wrap_device(0, Bd.data_ptr(), Bd.numel() * 4)
    hC = th.wrap_device(0, Cd.data_ptr(), Cd.numel() * 4)
    opts = nu.make_opts(k_chunk=kc)
    ooc_opts = nu.make_opts(schedule=SCHEDULES[args.schedule], k_chunk=kc,
                            shared_staging=-1 if args.no_shared_staging else 0)
    shared_peers = False
    if world > 1 and not args.no_shared_staging:
        # NEXT-1: siblings of a grid row / column share A / B panels over
        # NVLink; exchange the CUDA IPC handles of arenas and flag words.  If
        # any rank cannot export or import, every rank falls back to
        # unshared staging (no cross-process dependency is then planned).
        try:
            blob = t.peer_export(M, N, K, ooc_opts)
        except nu.NorthupError as ex:
            log(f"[rank {rank}] peer export failed ({ex}); falling back to unshared staging")
            blob = None
        blobs = [None] * world
        dist.all_gather_object(blobs, blob)
        ok = all(bl is not None for bl in blobs)
        if ok:
            try:
                for w, bl in enumerate(blobs):
                    if w != rank:
                        t.peer_import(w, bl)
            except nu.NorthupError as ex:
                log(f"[rank {rank}] peer import failed ({ex}); falling back to unshared staging")
                ok = False
        oks = [None] * world
        dist.all_gather_object(oks, ok)
        shared_peers = all(oks)
        if not shared_peers:
            ooc_opts = nu.make_opts(schedule=SCHEDULES[args.schedule], k_chunk=kc, shared_staging=-1)
    stream = torch.cuda.current_stream(dev)

    def barrier():
        torch.cuda.synchronize(dev)
        if dist is not None:
            dist.barrier()

    def max_over_ranks(x: float) -> float:
        if dist is None:
            return x
        v = torch.tensor([x], dtype=torch.float64, device=dev)
        dist.all_reduce(v, op=dist.ReduceOp.MAX)
        return float(v.item())

    def timed(fn, steps, warmup):
        """Device time (CUDA events on the torch stream bracketing synchronous
        calls, barrier + synchronize on both sides, max over ranks) and host
        wall time (perf_counter around the same calls, max over ranks)."""
        for _ in range(warmup):
            fn()
        barrier()
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(steps + 1)]
        w0 = time.perf_counter()
        evs[0].record(stream)
        for i in range(steps):
            fn()
            evs[i + 1].record(stream)
        barrier()
        wall = (time.perf_counter() - w0) * 1e3
        per = [evs[i].elapsed_time(evs[i + 1]) for i in range(steps)]
        return max_over_ranks(evs[0].elapsed_time(evs[-1])), max_over_ranks(wall), per

    ooc_stats, hbm_stats = {}, {}
    GM, GN = (M, N) if world > 1 else (m, n)

    def step_ooc():
        ooc_stats.update(t.gemm(Ab, Bb, Cb, GM, GN, K, ooc_opts))

    def step_hbm():
        hbm_stats.update(th.gemm(hA, hB, hC, m, n, K, opts))

    with ClockSampler(local_rank) as clk:
        for _ in range(args.warmup):      # warm both trees before either timed region
            step_ooc()
        nl0 = kernel_launches()
        t_ooc, wall_ooc, per_ooc = timed(step_ooc, args.steps, 0)
        launches_timed = kernel_launches() - nl0
        plan_ms_ooc = float(ooc_stats.get("t_plan_ms", 0.0))
        t_hbm, wall_hbm, per_hbm = timed(step_hbm, args.steps, args.warmup)
        # the dominant kernel, live: events around each GEMM kernel of the in-HBM
        # leaf on this stream (same operands, same panels)
        leaf_ms = leaf_kernel_ms(Ad, Bd, Cd, kc, stream, reps=1 if world > 1 else 2)
    ck = clk.summary()
    c_hbm = Cd.cpu().numpy()
    c_ooc = c.copy()
    bitwise_cross_tier = bool(np.array_equal(c_hbm, c_ooc))
    # the leaf on device pointers (northup_leaf_gemm) against the CS4 tree: same bits
    Cd2 = torch.empty_like(Cd)
    nu.leaf_gemm(Ad, Bd, Cd2, k_chunk=kc, stream=stream)
    torch.cuda.synchronize(dev)
    bitwise_tree_vs_leaf = bool(torch.equal(Cd, Cd2))
    del Cd2
    # the other splits of the leaf (R22), in-HBM rate only: npass = 4
    # adds lo.lo (4 MMAs per 16 k); npass = 1 is hi.hi alone (fails the bound)
    split_rates = {}
    if not args.quick or world == 1:
        for npass in (4, 1):
            e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
            nu.leaf_gemm(Ad, Bd, Cd, k_chunk=kc, npass=npass, stream=stream)
            e0.record(stream)
            nu.leaf_gemm(Ad, Bd, Cd, k_chunk=kc, npass=npass, stream=stream)
            e1.record(stream)
            torch.cuda.synchronize(dev)
            split_rates[f"npass{npass}"] = round(2.0 * m * n * K / (e0.elapsed_time(e1) * 1e-3) / 1e12, 3)
    # BJ configs[1] reference point: the 8192^3 GEMM resident in HBM, same leaf
    A2 = torch.rand((8192, 8192), device=dev) * 2 - 1
    B2 = torch.rand((8192, 8192), device=dev) * 2 - 1
    C2 = torch.empty((8192, 8192), device=dev)
    t_c2, _, _ = timed(lambda: nu.leaf_gemm(A2, B2, C2, k_chunk=kc, stream=stream), 5, 3)
    cfg2_tflops = 2.0 * 8192 ** 3 / (t_c2 / 5 * 1e-3) / 1e12
    del A2, B2, C2
    # staging evidence (untimed): one call in timing mode for per-stream busy
    # times, and the link bandwidth this GPU gets for pinned copies
    tim = t.gemm(Ab, Bb, Cb, GM, GN, K, nu.make_opts(schedule=ooc_opts.schedule, k_chunk=kc, collect_timing=True,
                                                     shared_staging=ooc_opts.shared_staging))
    pcie = measure_pcie(dev)
    replicate_ms = None
    if world > 1 and args.replicate:
        from paper_conf_ipps_chey19_b200.dist import gather_regions
        creg = torch.from_numpy(c).to(dev) if args.dist_backend == "nccl" else torch.from_numpy(c.copy())
        barrier()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        e0.record(stream)
        full = gather_regions(creg, M, N, K, rank, world)
        e1.record(stream)
        barrier()
        replicate_ms = e0.elapsed_time(e1)
        ok = bool(torch.equal(full[r0:r1, c0:c1].cpu(), torch.from_numpy(c)))
        del full
        replicate_ms = (replicate_ms, ok)

    flops_total = 2.0 * M * N * K
    ms_ooc = t_ooc / args.steps
    ms_hbm = t_hbm / args.steps
    value = flops_total / (ms_ooc * 1e-3) / 1e12
    in_hbm = flops_total / (ms_hbm * 1e-3) / 1e12
    e2e = flops_total / (wall_ooc / args.steps * 1e-3) / 1e12
    peaks = measured_peaks()
    # burst peak when the timed region ran at full clocks (a short step, no power
    # cap), the sustained one when the power cap pulled the clocks down
    at_max = bool(ck.get("sm_mhz") and ck.get("sm_max_mhz") and ck["sm_mhz"] >= 0.95 * ck["sm_max_mhz"])
    peak_kind = "burst" if at_max else "sustained"
    p_bf16 = peaks["bf16_burst"] if at_max else peaks["bf16_sustained"]
    # leaf split (R22): three fp16 MMAs per useful MAC (hi.hi, hi.lo,
    # lo.hi); fp16 and bf16 share the dense tensor rate -> P_eff = P_bf16 / 3
    p_eff = p_bf16 / 3.0
    kc_eff = kc or 2048
    flops_per_launch = 2.0 * m * min(n, 32768) * min(K, kc_eff)
    kern_ms = statistics.mean(leaf_ms) if leaf_ms else float("nan")
    achieved = flops_per_launch / (kern_ms * 1e-3) / 1e12
    launches_per_leaf = -(-K // kc_eff) * (-(-n // 32768))
    traffic = tensor_active = None
    tp = os.path.join(ROOT, "profiles", "leaf_traffic.json")
    if os.path.exists(tp):
        with open(tp) as f:
            tj = json.load(f)
        if (tj.get("M"), tj.get("N"), tj.get("launch_K")) == (m, min(n, 32768), min(K, kc_eff)):
            traffic = tj.get("dram_bytes")
            tensor_active = tj.get("tensor_pipe_active_pct")
    step_ms_tim = max(1e-9, float(tim.get("t_total_ms", ms_ooc)))
    result = None
    if rank == 0:
        cpu = None
        if world == 1 and not args.no_cpu_baseline:
            os.sched_setaffinity(0, all_cpus)          # the oracle gets every host core
            cpu = cpu_baseline(dict(cfg, M=m, N=n), a, b, c_ooc, args.cpu_budget)
        result = {
            "metric": METRIC,
            "value": round(value, 3),
            "unit": "TFLOP/s",
            "n_gpus": world,
            "steps": args.steps,
            "warmup": args.warmup,
            "ms_per_step": round(ms_ooc, 3),
            "higher_is_better": True,
            "scaling": "strong" if world > 1 else "weak",
            "vs_baseline": None,
            "dtype": "f32 (tcgen05 kind::f16 on a scaled fp16 hi/lo split, 3 MMAs per 16 k, fp32 accumulate)",
            "data": "synthetic (counter-hash uniform [-1,1) fp32, seed = config index)",
            "config": {
                "workload": f"{name}: {cfg['desc']}" + (" [quick: /4 sizes]" if args.quick else ""),
                "M": M, "N": N, "K": K, "hbm_cap_bytes": cfg["cap"], "k_panel": kc or 2048,
                "tmem_acc_chunk": 256,
                "region_per_gpu": [m, n, K],
                "parallelism": f"C subtrees {nu.partition(world, M, N)} over {world} GPU(s)" if world > 1 else "1 GPU",
                "schedule": {1: "S1", 2: "S2 (drain tail)", 3: "queue", 4: "S2B (B-first)"}.get(
                    ooc_stats.get("schedule"), "auto"),
                "bfirst_rows": ooc_stats.get("bfirst_rows"),
                "shared_staging": bool(ooc_stats.get("shared_staging")),
                "shared_staging_peers": "CUDA IPC (multi-process siblings)" if shared_peers else None,
                "blocks": [ooc_stats.get("bm"), ooc_stats.get("bn"), ooc_stats.get("bk")],
                "drain_tail_k": ooc_stats.get("tail_k"), "drain_strips": ooc_stats.get("strips"),
                "hbm_footprint_bytes": ooc_stats.get("hbm_peak_bytes"),
                "numa": numa,
                "links_at_finalize": t.link_info(),
                "l2": "inputs (>= 4 GiB each) exceed the 126 MB L2; no flush needed",
                "value_basis": "out-of-core: northup_gemm from pinned HOST buffers through the tree, every "
                               "H2D/D2H inside the step; CUDA events on the calling stream bracketing the "
                               "synchronous calls, max over ranks",
            },
            "e2e": {"value": round(e2e, 3), "unit": "TFLOP/s",
                    "h2d_bytes_per_step": int(ooc_stats.get("bytes_h2d", 0)),
                    "d2h_bytes_per_step": int(ooc_stats.get("bytes_d2h", 0)),
                    "p2p_bytes_per_step": int(ooc_stats.get("bytes_p2p", 0)),
                    "ms_per_step": round(wall_ooc / args.steps, 3),
                    "leaf_launches_per_step": int(ooc_stats.get("leaf_launches", 0)),
                    "basis": "the same northup_gemm calls timed by the host clock (planning and issue included)"},
            "in_hbm": {"value": round(in_hbm, 3), "unit": "TFLOP/s", "ms_per_step": round(ms_hbm, 3),
                       "basis": "single-node HBM tree (CS4): northup_gemm on operands resident in HBM, same "
                                "leaf and K-panel sequence (reading R16)",
                       "split_variants_tflops": split_rates},
            "slowdown_pct_vs_in_hbm": round(100.0 * (ms_ooc / ms_hbm - 1.0), 2),
            "cfg2_in_hbm_tflops": round(cfg2_tflops, 3),
            "slowdown_pct_vs_cfg2_in_hbm": round(100.0 * (cfg2_tflops / (value / world) - 1.0), 2),
            "runtime_overhead": {
                "plan_ms": round(plan_ms_ooc, 3),
                "plan_pct_of_step": round(100.0 * plan_ms_ooc / ms_ooc, 3),
                "host_vs_device_ms_per_step": round((wall_ooc - t_ooc) / args.steps, 3),
                "paper": "P:367: runtime overhead below 1 %",
            },
            "breakdown": {   # Fig. 7/8 analogue: stream busy shares of one out-of-core step
                "step_ms": round(step_ms_tim, 3),
                "compute_pct": round(100.0 * tim.get("t_compute_ms", 0.0) / step_ms_tim, 1),
                "h2d_pct": round(100.0 * tim.get("t_h2d_ms", 0.0) / step_ms_tim, 1),
                "d2h_pct": round(100.0 * tim.get("t_d2h_ms", 0.0) / step_ms_tim, 1),
                "p2p_pct": round(100.0 * tim.get("t_p2p_ms", 0.0) / step_ms_tim, 1),
                "exposed_transfer_pct": round(100.0 * max(0.0, step_ms_tim - tim.get("t_compute_ms", 0.0))
                                              / step_ms_tim, 1),
                "basis": "CUDA events around every op of one untimed call (collect_timing); busy = sum of "
                         "op durations per stream; exposed = step - compute busy",
            },
            "staging": {
                "pcie_measured": pcie,
                "h2d_busy_gbs": round(tim["bytes_h2d"] / (tim["t_h2d_ms"] * 1e6), 2) if tim.get("t_h2d_ms") else None,
                "d2h_busy_gbs": round(tim["bytes_d2h"] / (tim["t_d2h_ms"] * 1e6), 2) if tim.get("t_d2h_ms") else None,
                "h2d_avg_gbs_over_step": round(ooc_stats.get("bytes_h2d", 0) / (ms_ooc * 1e6), 2),
                "d2h_avg_gbs_over_step": round(ooc_stats.get("bytes_d2h", 0) / (ms_ooc * 1e6), 2),
                "busy_ms": {k: round(tim.get(k, 0.0), 2) for k in ("t_h2d_ms", "t_compute_ms", "t_d2h_ms", "t_p2p_ms")},
                "basis": "busy = sum of the copy-stream op durations (CUDA events, one untimed call in timing mode)"},
            "e2e_roofline": None,
            "replicate": None if replicate_ms is None else {
                "ms": round(replicate_ms[0], 3), "region_roundtrip_ok": replicate_ms[1],
                "backend": args.dist_backend,
                "bytes_per_gpu_received": 4 * (M * N - m * n)},
            "paper_context": {"avg_ooc_slowdown_pct": 17, "dmm_ooc_gap_pct": 5,
                              "note": "APU + SSD, OpenCL fp32 (PAPER.md P:10, P:381); context only"},
            "roofline": {"bound": "tensor", "achieved": round(achieved, 3),
                         "peak": round(p_eff, 3), "unit": "TFLOP/s",
                         "frac": round(achieved / p_eff, 4), "traffic": traffic,
                         "peak_basis": (f"useful-flop ceiling of the split P_bf16 / 3 (three fp16 MMAs per useful "
                                        f"MAC; fp16 = bf16 dense rate): P_bf16 = {peaks['source']} bf16 "
                                        f"{peak_kind} {p_bf16} TF/s (burst if the timed region's median SM clock "
                                        f"was >= 0.95 x max, else sustained)"),
                         "kernel": "nu::leaf::x3::leaf_x3_kernel",
                         "launch": [m, min(n, 32768), min(K, kc_eff)], "launches_per_leaf_call": launches_per_leaf,
                         "flops_per_launch": flops_per_launch, "ms_per_launch": round(kern_ms, 3),
                         "launches_timed": len(leaf_ms),
                         "tensor_pipe_active_pct_ncu": tensor_active,
                         "achieved_basis": "useful flops 2 m n k of one K-panel launch / its CUDA-event duration "
                                           "(events recorded by the library around each GEMM kernel on the torch "
                                           "stream, in-HBM operands)",
                         "traffic_basis": "ncu --set full dram__bytes_read+write of one reduce-add launch "
                                          "(profiles/leaf_traffic.json); algorithmic bytes of such a launch "
                                          f"= split A/B panel + C read + C write = "
                                          f"{4 * (m + min(n, 32768)) * min(K, kc_eff) + 8 * m * min(n, 32768):.3e}"
                                          + (f" (traffic / algorithmic = {traffic / (4 * (m + min(n, 32768)) * min(K, kc_eff) + 8 * m * min(n, 32768)):.2f})"
                                             if traffic else "")},
            "gpu_launches": launches_timed * world,
            "gpu_launches_basis": "library kernel launches (northup_debug_kernel_launches) during the timed "
                                  "out-of-core steps on this rank x ranks",
            "parity": {"bitwise_in_hbm_vs_out_of_core": bitwise_cross_tier,
                       "bitwise_tree_vs_leaf": bitwise_tree_vs_leaf},
            "clocks": ck,
        }
        rl = ooc_roofline(2.0 * m * n * K, int(ooc_stats.get("bytes_h2d", 0)),
                          int(ooc_stats.get("bytes_d2h", 0)), p_eff, pcie)
        v_gpu = 2.0 * m * n * K / (ms_ooc * 1e-3) / 1e12
        rl.update(achieved=round(v_gpu, 3), frac=round(v_gpu / rl["peak"], 4),
                  basis="per GPU: out-of-core TF/s of this GPU's region / min(P_eff, BW_e x I_e) (S§8(d))")
        result["e2e_roofline"] = rl
        if cpu is not None:
            result["cpu_baseline"] = {k: cpu[k] for k in ("value", "unit", "cores", "kind", "sample")}
            for k in ("cpu_model", "numa_nodes", "single_core_value"):
                result["cpu_baseline"][k] = cpu.get(k)
            result["parity"]["oracle_normwise_err_rows"] = cpu.get("gpu_normwise_err_on_sample")
            result["parity"]["oracle_ok"] = cpu.get("gpu_parity_ok")
    th.destroy()
    t.destroy()
    return result


# ------------------------------------------------------------ HotSpot-2D
def run_hotspot(args, rank: int, world: int, local_rank: int):
    """NEXT-3: HotSpot-2D over the tree.  value = out-of-core (HOST -> HBM (8 GiB
    cap) -> SMEM through northup_hotspot with pinned host grids); in_hbm = the
    single-node HBM tree with the grids resident.  Unit: cell updates per second."""
    import numpy as np
    import torch
    import nugen
    import paper_conf_ipps_chey19_b200 as nu
    from oracle import hotspot as ohs

    dev = torch.device("cuda", local_rank)
    torch.cuda.set_device(dev)
    R, C, iters, cap = HOTSPOT["R"], HOTSPOT["C"], HOTSPOT["iters"], HOTSPOT["cap"]
    if args.quick:
        R, C, cap = R // 4, C // 4, cap // 16
    t, _ = nu.host_tree(1, cap, devices=[local_rank])
    t.finalize()
    Tb, Pb, Ob = t.alloc(4 * R * C, 0), t.alloc(4 * R * C, 0), t.alloc(4 * R * C, 0)
    T, P, O = host_array(Tb.ptr, R, C), host_array(Pb.ptr, R, C), host_array(Ob.ptr, R, C)
    nugen.fill(R, C, 6, nugen.MAT_T, "temp", out=T)
    nugen.fill(R, C, 6, nugen.MAT_P, "power", out=P)
    th = nu.hbm_tree(local_rank)
    th.finalize()
    Td, Pd = torch.from_numpy(T).to(dev), torch.from_numpy(P).to(dev)
    Od = torch.empty_like(Td)
    hT, hP, hO = (th.wrap_device(0, x.data_ptr(), x.numel() * 4) for x in (Td, Pd, Od))
    stream = torch.cuda.current_stream(dev)
    st_h, st_o = {}, {}

    def timed(fn, steps, warmup):
        for _ in range(warmup):
            fn()
        torch.cuda.synchronize(dev)
        evs = [torch.cuda.Event(enable_timing=True) for _ in range(steps + 1)]
        evs[0].record(stream)
        for i in range(steps):
            fn()
            evs[i + 1].record(stream)
        torch.cuda.synchronize(dev)
        return evs[0].elapsed_time(evs[-1]), [evs[i].elapsed_time(evs[i + 1]) for i in range(steps)]

    with ClockSampler(local_rank) as clk:
        t_h, per_h = timed(lambda: st_h.update(th.hotspot(hT, hP, hO, R, C, iters)), args.steps, args.warmup)
        t_o, per_o = timed(lambda: st_o.update(t.hotspot(Tb, Pb, Ob, R, C, iters)), args.steps, args.warmup)
    # Fig. 7/8 analogue (untimed): one out-of-core call in timing mode, per-stream busy time
    tim = t.hotspot(Tb, Pb, Ob, R, C, iters, nu.hotspot_opts(collect_timing=1))
    torch.cuda.synchronize(dev)
    o_hbm = Od.cpu().numpy()
    bitwise = bool(np.array_equal(o_hbm, O))
    cells = float(R) * C * iters
    ms_h, ms_o = t_h / args.steps, t_o / args.steps
    in_hbm = cells / (ms_h * 1e-3) / 1e9
    value = cells / (ms_o * 1e-3) / 1e9
    launches = st_h.get("leaf_launches", 0)
    leaf_ms = statistics.mean(per_h) / max(1, launches)
    li = st_h.get("bk", 8)
    flops_per_launch = HS_FLOPS_PER_UPDATE * float(R) * C * li
    achieved = flops_per_launch / (leaf_ms * 1e-3) / 1e12
    ck = clk.summary()
    f_max = (ck.get("sm_max_mhz") or 1965.0) * 1e6
    peak = 2 * N_SMS * FP32_LANES_PER_SM * f_max / 1e12     # fp32 FMA = 2 flops per lane per clock
    # parity: sampled blocks against the fp64 oracle (window of border `iters`)
    k64 = ohs.coeffs(R, C)
    rng = np.random.default_rng(11)
    worst, tmax = 0.0, 0.0
    samples = [(0, 0), (R - 32, C - 32)] + [(int(y), int(x)) for y, x in
                                            zip(rng.integers(0, R - 32, 2), rng.integers(0, C - 32, 2))]
    t0 = time.perf_counter()
    for (y0, x0) in samples:
        wy0, wx0 = max(0, y0 - iters), max(0, x0 - iters)
        wy1, wx1 = min(R, y0 + 32 + iters), min(C, x0 + 32 + iters)
        tw = T[wy0:wy1, wx0:wx1].astype(np.float64)
        pw = P[wy0:wy1, wx0:wx1].astype(np.float64)
        for _ in range(iters):
            tw = ohs._window_step(tw, pw, wy0, wx0, R, C, k64)
        ref = tw[y0 - wy0:y0 - wy0 + 32, x0 - wx0:x0 - wx0 + 32]
        worst = max(worst, float(np.abs(O[y0:y0 + 32, x0:x0 + 32] - ref).max()))
        tmax = max(tmax, float(np.abs(ref).max()))
    cpu_s = time.perf_counter() - t0
    cpu_cells = sum((min(R, y + 32 + iters) - max(0, y - iters)) * (min(C, x + 32 + iters) - max(0, x - iters))
                    for y, x in samples) * iters
    tol = ohs.tolerance(iters, tmax)
    # the link rates measured in this run with both directions active (as for the GEMM lines):
    # T and P windows cross H2D once per pass while the finished blocks drain D2H
    pcie = measure_pcie(dev)
    t_h2d = st_o.get("bytes_h2d", 0) / (pcie["bidir_h2d_gbs"] * 1e9)
    t_d2h = st_o.get("bytes_d2h", 0) / (pcie["bidir_d2h_gbs"] * 1e9)
    pcie_gcups = cells / max(t_h2d, t_d2h, 1e-12) / 1e9
    pcie_bound = "pcie_h2d" if t_h2d >= t_d2h else "pcie_d2h"
    # DRAM bytes per launch from the committed ncu capture of the same launch shape
    hs_traffic = None
    tp = os.path.join(ROOT, "profiles", "hotspot_traffic.json")
    if os.path.exists(tp):
        with open(tp) as f:
            tj = json.load(f)
        if (tj.get("R"), tj.get("C"), tj.get("leaf_iters")) == (R, C, st_h.get("bk", 8)):
            hs_traffic = tj.get("dram_bytes")
    result = {
        "metric": "out-of-core HotSpot-2D cell updates/s (S§8(f) NEXT-3); % slowdown vs in-HBM; roofline frac",
        "value": round(value, 3), "unit": "Gcell-updates/s", "n_gpus": 1, "steps": args.steps,
        "warmup": args.warmup, "ms_per_step": round(ms_o, 3), "higher_is_better": True, "scaling": "weak",
        "vs_baseline": None, "dtype": "f32 (fixed FADD/FFMA sequence, RH4)",
        "data": "synthetic (counter-hash temperature 330 +- 10 K, power [0, 0.5))",
        "config": {"workload": "hotspot: " + HOTSPOT["desc"] + (" [quick: /4 sizes]" if args.quick else ""),
                   "rows": R, "cols": C, "iters": iters, "hbm_cap_bytes": cap,
                   "block": st_o.get("bm"), "halo_iters_per_visit": st_o.get("bk"),
                   "leaf_iters_per_launch": li,
                   "l2": "grids (4 GiB each) exceed the 126 MB L2; no flush needed"},
        "in_hbm": {"value": round(in_hbm, 3), "unit": "Gcell-updates/s", "ms_per_step": round(ms_h, 3)},
        "e2e": {"value": round(value, 3), "unit": "Gcell-updates/s",
                "h2d_bytes_per_step": int(st_o.get("bytes_h2d", 0)),
                "d2h_bytes_per_step": int(st_o.get("bytes_d2h", 0)), "ms_per_step": round(ms_o, 3),
                "leaf_launches_per_step": int(st_o.get("leaf_launches", 0)),
                "pcie_roofline_gcups": round(pcie_gcups, 1), "pcie_measured": pcie},
        "slowdown_pct_vs_in_hbm": round(100.0 * (ms_o / ms_h - 1.0), 2),
        "e2e_roofline": {"bound": pcie_bound if pcie_gcups < in_hbm else "in_hbm",
                         "peak": round(min(pcie_gcups, in_hbm), 1), "unit": "Gcell-updates/s",
                         "frac": round(value / min(pcie_gcups, in_hbm), 4),
                         "terms": {"pcie_h2d": round(cells / max(t_h2d, 1e-12) / 1e9, 1),
                                   "pcie_d2h": round(cells / max(t_d2h, 1e-12) / 1e9, 1),
                                   "in_hbm": round(in_hbm, 1)},
                         "basis": "min(plan's H2D bytes / BW_h2d, D2H bytes / BW_d2h, the in-HBM rate), BW = "
                                  "pinned copies measured in this run with both directions active; T and P "
                                  "windows cross PCIe once per pass"},
        "breakdown": {k.replace("t_", "").replace("_ms", "_busy_ms"): round(tim.get(k, 0.0), 2)
                      for k in ("t_h2d_ms", "t_compute_ms", "t_d2h_ms")} | {
            "h2d_busy_gbs": round(tim["bytes_h2d"] / (tim["t_h2d_ms"] * 1e6), 2) if tim.get("t_h2d_ms") else None,
            "basis": "CUDA events around every op of one untimed out-of-core call (collect_timing); busy = sum "
                     "of op durations per stream"},
        "paper_context": {"hotspot_ooc_gap_pct": 15, "note": "APU + SSD vs DRAM (PAPER.md P:381); context only"},
        "roofline": {"bound": "alu", "achieved": round(achieved, 3), "peak": round(peak, 3), "unit": "TFLOP/s",
                     "frac": round(achieved / peak, 4), "traffic": hs_traffic,
                     "peak_basis": f"dense fp32 peak: {N_SMS} SMs x {FP32_LANES_PER_SM} lanes x 2 flops (FMA) x "
                                   f"clocks.max.sm {f_max / 1e6:.0f} MHz",
                     "kernel": "nu::hs::hotspot_kernel_tma", "launch": [R, C, li],
                     "flops_per_launch": flops_per_launch,
                     "flops_basis": f"{HS_FLOPS_PER_UPDATE} flops per useful cell update (the update's "
                                    f"5 multiplies + 9 adds; the kernel issues 3 FADD + 6 FFMA) x R x C x "
                                    f"iterations per launch (halo recomputation not counted)",
                     "ms_per_launch": round(leaf_ms, 3), "launches_per_step": launches},
        "gpu_launches": int(launches * args.steps + st_o.get("leaf_launches", 0) * args.steps),
        "parity": {"bitwise_in_hbm_vs_out_of_core": bitwise,
                   "oracle_max_abs_err_sampled_blocks": worst, "oracle_tolerance": tol,
                   "oracle_ok": bool(worst <= tol), "sampled_blocks": len(samples)},
        "clocks": ck,
        "cpu_baseline": {"value": round(cpu_cells / cpu_s / 1e9, 6), "unit": "Gcell-updates/s", "cores": 1,
                         "kind": "oracle",
                         "sample": f"{len(samples)} 32x32 blocks with {iters}-cell borders x {iters} iterations "
                                   f"(fp64 numpy window sweeps), {cpu_s:.1f} s"},
    }
    th.destroy()
    t.destroy()
    return result


# --------------------------------------------------------------- FILE root
def measure_disk(d: str, nbytes: int = 1 << 30) -> dict:
    """Sequential O_DIRECT write then read of one file on the bench's file
    system (GB/s): the disk term of the FILE-root roofline (S§8(d))."""
    import mmap
    path = os.path.join(d, "disk_probe.bin")
    chunk = 64 << 20
    buf = mmap.mmap(-1, chunk)                      # page-aligned (O_DIRECT)
    buf.write(os.urandom(1 << 20) * (chunk >> 20))
    flags = getattr(os, "O_DIRECT", 0)
    out = {"how": f"O_DIRECT {nbytes >> 20} MiB sequential in {chunk >> 20} MiB requests, fsync before stopping the clock"}
    fd = os.open(path, os.O_CREAT | os.O_WRONLY | os.O_TRUNC | flags, 0o644)
    t0 = time.perf_counter()
    for off in range(0, nbytes, chunk):
        os.pwrite(fd, buf, off)
    os.fsync(fd)
    out["write_gbs"] = round(nbytes / (time.perf_counter() - t0) / 1e9, 3)
    os.close(fd)
    fd = os.open(path, os.O_RDONLY | flags)
    t0 = time.perf_counter()
    for off in range(0, nbytes, chunk):
        os.preadv(fd, [buf], off)
    out["read_gbs"] = round(nbytes / (time.perf_counter() - t0) / 1e9, 3)
    os.close(fd)
    os.unlink(path)
    out["o_direct"] = bool(flags)
    return out


def run_file(args, rank: int, world: int, local_rank: int):
    """S§8(a) a3 / NEXT-4: the GEMM with A, B, C in files on the box's disk:
    value = FILE -> HOST staging -> HBM (8 GiB cap) -> SMEM/TMEM; the direct
    edge FILE -> HBM (pinned bounce, or cuFile with NORTHUP_CUFILE=1) beside it;
    roofline against the measured disk read / write bandwidth."""
    import shutil
    import tempfile
    import numpy as np
    import torch
    import nugen
    import oracle
    import paper_conf_ipps_chey19_b200 as nu

    dev = torch.device("cuda", local_rank)
    torch.cuda.set_device(dev)
    n = args.file_size or 32768
    if args.quick:
        n //= 4
    M = N = K = n
    panel = 2048 if K >= 2048 else K
    base = args.file_dir or os.environ.get("NORTHUP_BENCH_FILE_DIR") or "/tmp"
    free = shutil.disk_usage(base).free
    if free < 6 * 4 * n * n:
        return {"metric": METRIC, "unavailable": f"{base}: {free >> 30} GiB free < {6 * 4 * n * n >> 30} GiB"}
    d = tempfile.mkdtemp(dir=base, prefix="northup_bench_")
    try:
        seed = 4
        a = nugen.fill(M, K, seed, nugen.MAT_A)
        b = nugen.fill(K, N, seed, nugen.MAT_B)
        a.tofile(f"{d}/A.bin")
        b.tofile(f"{d}/B.bin")
        t0 = time.perf_counter()
        nu.file_tile_kpanels(f"{d}/A.bin", f"{d}/A_t.bin", M, K, panel)     # R15, outside the timing
        pre_s = time.perf_counter() - t0
        os.unlink(f"{d}/A.bin")
        disk = measure_disk(d)
        runs = {}
        for kind in ("staging", "direct"):
            t = nu.Tree()
            root = t.add_node(-1, nu.NU_FILE)
            parent = t.add_node(root, nu.NU_HOST, -1, 0) if kind == "staging" else root
            h = t.add_node(parent, nu.NU_HBM, local_rank, 8 * GiB)
            t.add_node(h, nu.NU_SMEM, local_rank, 227 * 1024, nu.NU_PROC_SM100)
            t.finalize()
            fa = t.open_file(0, f"{d}/A_t.bin", 4 * M * K)
            fb = t.open_file(0, f"{d}/B.bin", 4 * K * N)
            fc = t.open_file(0, f"{d}/C_{kind}.bin", 4 * M * N)
            o = nu.make_opts(a_panel_k=panel)
            for _ in range(max(1, args.warmup)):
                t.gemm(fa, fb, fc, M, N, K, o)
            ms, st = [], {}
            for _ in range(args.steps):
                t0 = time.perf_counter()
                st = t.gemm(fa, fb, fc, M, N, K, o)     # synchronous: C durable in its file
                ms.append((time.perf_counter() - t0) * 1e3)
            t.destroy()
            c = np.fromfile(f"{d}/C_{kind}.bin", dtype=np.float32).reshape(M, N)
            rows = np.arange(0, M, max(1, M // 16))
            ref = oracle.gemm_rows(a, b, rows)
            e, _ = oracle.normwise_err(np.ascontiguousarray(c[rows]), ref,
                                       oracle.row_norms(np.ascontiguousarray(a[rows])), oracle.col_norms(b))
            runs[kind] = {"ms_per_step": round(statistics.mean(ms), 3),
                          "tflops": round(2.0 * M * N * K / (statistics.mean(ms) * 1e-3) / 1e12, 3),
                          "file_read_bytes": int(st["bytes_file_read"]), "file_write_bytes": int(st["bytes_file_write"]),
                          "io_busy_ms": round(st["t_io_ms"], 1), "file_direct_mode": int(st["file_direct_mode"]),
                          "normwise_err_16_rows": e}
        peaks = measured_peaks()
        p_eff = peaks["bf16_sustained"] / 3.0
        st = runs["staging"]
        t_disk = st["file_read_bytes"] / (disk["read_gbs"] * 1e9) + st["file_write_bytes"] / (disk["write_gbs"] * 1e9)
        disk_term = 2.0 * M * N * K / t_disk / 1e12
        bound = "disk" if disk_term < p_eff else "tensor"
        peak = min(disk_term, p_eff)
        value = st["tflops"]
        return {
            "metric": METRIC, "value": value, "unit": "TFLOP/s", "n_gpus": 1, "steps": args.steps,
            "warmup": args.warmup, "ms_per_step": st["ms_per_step"], "higher_is_better": True, "scaling": "weak",
            "vs_baseline": None, "dtype": "f32 (tcgen05 kind::f16 on a scaled fp16 hi/lo split, fp32 accumulate)",
            "data": "synthetic (counter-hash uniform [-1,1) fp32 in files on the box's disk)",
            "config": {"workload": f"file-root: {M}^3 fp32, FILE (no NVMe on the box: virtio disk, {base}) -> "
                                   f"HOST staging -> HBM (8 GiB cap) -> SMEM/TMEM, 1 GPU",
                       "M": M, "N": N, "K": K, "a_layout": f"K-panel-major, panel {panel} (R15)",
                       "preprocess_s": round(pre_s, 2)},
            "e2e": {"value": value, "unit": "TFLOP/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0,
                    "file_read_bytes_per_step": st["file_read_bytes"],
                    "file_write_bytes_per_step": st["file_write_bytes"],
                    "basis": "host clock around synchronous northup_gemm calls (C written and fdatasync'ed)"},
            "runs": runs, "disk": disk,
            "file_roofline": {"bound": bound, "peak": round(peak, 3), "unit": "TFLOP/s",
                              "terms": {"tensor": round(p_eff, 3), "disk": round(disk_term, 3)},
                              "achieved": value, "frac": round(value / peak, 4),
                              "basis": "min(P_eff, 2MNK / (file bytes read / disk read GB/s + file bytes written "
                                       "/ disk write GB/s)); read and write share the device"},
            "parity": {"oracle_ok": all(r["normwise_err_16_rows"] <= 1e-5 for r in runs.values())},
        }
    finally:
        shutil.rmtree(d, ignore_errors=True)


# --------------------------------------------------------------- reference
def run_reference(args):
    """The fp64 CPU oracle as the reference arm (bounded sample per step)."""
    import numpy as np
    import nugen
    import oracle
    name = args.config or "cfg3"
    cfg = dict(CONFIGS[name])
    if args.quick:
        cfg.update(M=cfg["M"] // 4, N=cfg["N"] // 4, K=cfg["K"] // 4)
    M, N, K = cfg["M"], cfg["N"], cfg["K"]
    seed = int(name[-1])
    cores = oracle.threads()
    b = nugen.fill(K, N, seed, nugen.MAT_B)
    rng = np.random.default_rng(7)

    def step(nrows):
        rows = np.sort(rng.choice(M, size=nrows, replace=False))
        a = np.empty((nrows, K), dtype=np.float32)
        for i, r in enumerate(rows):
            nugen.fill(1, K, seed, nugen.MAT_A, out=a[i:i + 1], i0=int(r), ncols=K)
        t0 = time.perf_counter()
        oracle.gemm(a, b)
        return time.perf_counter() - t0

    dt = step(cores)
    nrows = cores * max(1, int(args.ref_step_s / max(dt, 1e-3)))
    for _ in range(args.warmup):
        step(cores)
    times = [step(nrows) for _ in range(args.steps)]
    total = sum(times)
    flops = 2.0 * nrows * N * K * args.steps
    v = flops / total / 1e12
    return {
        "impl": "reference", "metric": METRIC, "value": round(v, 6), "unit": "TFLOP/s",
        "n_gpus": 1, "steps": args.steps, "warmup": args.warmup,
        "ms_per_step": round(1e3 * total / args.steps, 3), "higher_is_better": True,
        "scaling": "weak", "vs_baseline": None, "dtype": "f64", "data": "synthetic",
        "config": {"workload": f"{name}: {cfg['desc']}", "M": M, "N": N, "K": K},
        "cpu_baseline": {"value": round(v, 6), "unit": "TFLOP/s", "cores": cores, "kind": "oracle",
                         "sample": f"{nrows} full rows of C per step ({nrows}x{N}x{K})", **cpu_facts()},
        "e2e": {"value": round(v, 6), "unit": "TFLOP/s", "h2d_bytes_per_step": 0,
                "d2h_bytes_per_step": 0},
    }


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=5)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", default=None, choices=sorted(CONFIGS) + ["hotspot", "file"])
    ap.add_argument("--file-size", type=int, default=0, help="--config file: M = N = K (default 32768)")
    ap.add_argument("--file-dir", default=None, help="--config file: where the A, B, C files go")
    ap.add_argument("--k-chunk", type=int, default=2048)
    ap.add_argument("--schedule", default="auto", choices=sorted(SCHEDULES),
                    help="HOST -> HBM schedule (default: the planner's cost model)")
    ap.add_argument("--quick", action="store_true", help="sizes / 4 (smoke-testing the bench)")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--cpu-budget", type=float, default=15.0)
    ap.add_argument("--ref-step-s", type=float, default=5.0)
    ap.add_argument("--replicate", action="store_true",
                    help="N>1: after the timed steps, gather C to every GPU (S8e) and time it")
    ap.add_argument("--dist-backend", default="nccl", choices=["nccl", "gloo"],
                    help="process-group backend (gloo only for multi-rank tests on one GPU)")
    ap.add_argument("--no-shared-staging", action="store_true",
                    help="N>1: every rank loads its whole A/B strips over PCIe (no NVLink sharing)")
    ap.add_argument("--device-mod", type=int, default=0,
                    help="map LOCAL_RANK modulo this many GPUs (multi-rank tests on one GPU)")
    ap.add_argument("--no-numa-bind", action="store_true", help="do not bind ranks to their GPU's NUMA node")
    args = ap.parse_args()
    if args.warmup < 3:
        log("warning: the timing rules ask for >= 3 warm-up steps")
    if "WORLD_SIZE" not in os.environ and args.gpus > 1:
        # not under torchrun: start one rank per GPU ourselves (same command line)
        import socket
        with socket.socket() as sk:
            sk.bind(("127.0.0.1", 0))
            port = sk.getsockname()[1]
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={args.gpus}",
               "--master-addr", "127.0.0.1", f"--master-port={port}", os.path.abspath(__file__), *sys.argv[1:]]
        log("spawning:", " ".join(cmd))
        sys.exit(subprocess.call(cmd))
    world = int(os.environ.get("WORLD_SIZE", "1"))
    if world != args.gpus:
        log(f"error: --gpus {args.gpus} but WORLD_SIZE={world}; run one rank per GPU (torchrun "
            f"--nproc-per-node {args.gpus}) or drop --gpus")
        sys.exit(2)
    rank = int(os.environ.get("RANK", "0"))
    local_rank = int(os.environ.get("LOCAL_RANK", "0"))
    if args.device_mod > 0:          # test mode: several ranks share the visible GPUs
        local_rank %= args.device_mod

    if args.impl == "reference":
        if rank == 0 and args.config in ("hotspot", "file"):
            print(json.dumps({"impl": "reference", "unavailable": "the HotSpot-2D oracle is timed as cpu_baseline "
                                                                  "in the ours line (no separate reference arm)"}))
            return
        if rank == 0:
            print(json.dumps(run_reference(args)), flush=True)
        return

    if world > 1:
        # a sibling process that fails leaves its peers' streams waiting on its flag
        # words; end the run after 3 minutes instead of the library's 10
        os.environ.setdefault("NORTHUP_PEER_TIMEOUT_S", "180")
        import torch
        import torch.distributed as dist
        torch.cuda.set_device(local_rank)
        if args.dist_backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local_rank))
        else:
            dist.init_process_group(args.dist_backend)
    res = run_hotspot(args, rank, world, local_rank) if args.config == "hotspot" else \
        run_file(args, rank, world, local_rank) if args.config == "file" else \
        run_ours(args, rank, world, local_rank)
    if rank == 0 and res is not None:
        print(json.dumps(res), flush=True)
    if world > 1:
        import torch.distributed as dist
        dist.barrier()
        dist.destroy_process_group()


if __name__ == "__main__":
    main()
