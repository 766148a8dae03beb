"""paper_conf_ipps_chey19_b200 — B200-native Northup out-of-core recursive GEMM.

A thin ctypes binding over the C ABI of libnorthup.so (include/northup.h):
argument marshalling only.  Every step of the GEMM path (planning, staging,
the sm_100a leaf kernel) runs in the native library; there is no Python or
CPU fallback — if the library is missing, every call raises.

PyTorch is used only as plumbing: device memory (arenas, resident operands)
and CUDA streams, passed to the library as raw pointers.
"""
from __future__ import annotations

import ctypes
import os
import re

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.environ.get("NORTHUP_LIB_PATH") or os.path.join(_HERE, "libnorthup.so")
HEADER = os.path.join(os.path.dirname(_HERE), "include", "northup.h")

# status codes / enums (include/northup.h)
NU_OK, NU_EINVAL, NU_ENOMEM, NU_EIO, NU_ECUDA, NU_ENCCL, NU_ESTATE, NU_ENOTSUP = 0, -1, -2, -3, -4, -5, -6, -7
NU_FILE, NU_HOST, NU_HBM, NU_SMEM = 0, 1, 2, 3
NU_PROC_NONE, NU_PROC_SM100 = 0, 1
NU_SCHED_AUTO, NU_SCHED_S1, NU_SCHED_S2, NU_SCHED_QUEUE, NU_SCHED_S2B = 0, 1, 2, 3, 4
NU_OP_COPY, NU_OP_LEAF, NU_OP_ZERO, NU_OP_IO_READ, NU_OP_IO_WRITE, NU_OP_STENCIL = 0, 1, 2, 3, 4, 5
NU_OP_SPLIT_B = 6
STREAM_NAMES = {0: "h2d", 1: "compute", 2: "d2h", 3: "io", 4: "d2d"}
STATUS_NAMES = {0: "NU_OK", -1: "NU_EINVAL", -2: "NU_ENOMEM", -3: "NU_EIO", -4: "NU_ECUDA",
                -5: "NU_ENCCL", -6: "NU_ESTATE", -7: "NU_ENOTSUP"}
GiB = 1 << 30


class NorthupError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{STATUS_NAMES.get(code, code)}: {msg}")
        self.code = code


class NodeInfo(ctypes.Structure):
    _fields_ = [("node_id", ctypes.c_int), ("storage_type", ctypes.c_int),
                ("physical_id", ctypes.c_int), ("capacity", ctypes.c_uint64),
                ("used", ctypes.c_uint64), ("processor_type", ctypes.c_int),
                ("level", ctypes.c_int), ("is_leaf", ctypes.c_int), ("parent", ctypes.c_int),
                ("num_children", ctypes.c_int), ("block_bm", ctypes.c_int64),
                ("block_bn", ctypes.c_int64), ("block_bk", ctypes.c_int64)]


class GemmOpts(ctypes.Structure):
    _fields_ = [("schedule", ctypes.c_int), ("replicate_result", ctypes.c_int),
                ("k_chunk", ctypes.c_int64), ("npass", ctypes.c_int), ("resident", ctypes.c_int),
                ("collect_timing", ctypes.c_int), ("a_panel_k", ctypes.c_int64),
                ("graph", ctypes.c_int), ("shared_staging", ctypes.c_int),
                ("queue_tiles", ctypes.c_int), ("reserved", ctypes.c_int * 3)]


class Stats(ctypes.Structure):
    _fields_ = [("t_total_ms", ctypes.c_double), ("t_plan_ms", ctypes.c_double),
                ("t_h2d_ms", ctypes.c_double), ("t_compute_ms", ctypes.c_double),
                ("t_d2h_ms", ctypes.c_double), ("t_io_ms", ctypes.c_double),
                ("bytes_h2d", ctypes.c_uint64), ("bytes_d2h", ctypes.c_uint64),
                ("bytes_d2d", ctypes.c_uint64), ("bytes_file_read", ctypes.c_uint64),
                ("bytes_file_write", ctypes.c_uint64), ("leaf_launches", ctypes.c_int64),
                ("copies", ctypes.c_int64), ("ops", ctypes.c_int64), ("bm", ctypes.c_int64),
                ("bn", ctypes.c_int64), ("bk", ctypes.c_int64), ("tail_k", ctypes.c_int64),
                ("strips", ctypes.c_int64), ("schedule", ctypes.c_int), ("num_gpus", ctypes.c_int),
                ("hbm_peak_bytes", ctypes.c_uint64), ("graph_replayed", ctypes.c_int),
                ("shared_staging", ctypes.c_int), ("bytes_p2p", ctypes.c_uint64),
                ("t_p2p_ms", ctypes.c_double), ("tasks", ctypes.c_int64),
                ("tasks_stolen", ctypes.c_int64), ("file_direct_mode", ctypes.c_int),
                ("bfirst_rows", ctypes.c_int)]

    def as_dict(self) -> dict:
        return {k: getattr(self, k) for k, _ in self._fields_}


class HotspotCoeffs(ctypes.Structure):
    _fields_ = [("cap_1", ctypes.c_float), ("rx_1", ctypes.c_float), ("ry_1", ctypes.c_float),
                ("rz_1", ctypes.c_float), ("amb", ctypes.c_float)]


class HotspotOpts(ctypes.Structure):
    _fields_ = [("block", ctypes.c_int64), ("halo", ctypes.c_int64), ("leaf_iters", ctypes.c_int),
                ("collect_timing", ctypes.c_int), ("reserved", ctypes.c_int * 4)]


class Op(ctypes.Structure):
    _fields_ = [("op", ctypes.c_int), ("worker", ctypes.c_int), ("stream", ctypes.c_int),
                ("accumulate", ctypes.c_int), ("src_buf", ctypes.c_int), ("dst_buf", ctypes.c_int),
                ("a_buf", ctypes.c_int), ("b_buf", ctypes.c_int), ("c_buf", ctypes.c_int),
                ("src_off", ctypes.c_int64), ("dst_off", ctypes.c_int64),
                ("src_ld", ctypes.c_int64), ("dst_ld", ctypes.c_int64), ("rows", ctypes.c_int64),
                ("cols", ctypes.c_int64), ("a_off", ctypes.c_int64), ("b_off", ctypes.c_int64),
                ("c_off", ctypes.c_int64), ("lda", ctypes.c_int64), ("ldb", ctypes.c_int64),
                ("ldc", ctypes.c_int64), ("m", ctypes.c_int64), ("n", ctypes.c_int64),
                ("k", ctypes.c_int64), ("ndeps", ctypes.c_int), ("deps", ctypes.c_int * 16)]

    def as_dict(self) -> dict:
        d = {k: getattr(self, k) for k, _ in self._fields_ if k != "deps"}
        d["deps"] = [self.deps[i] for i in range(self.ndeps)]
        return d


class PlanBuf(ctypes.Structure):
    _fields_ = [("kind", ctypes.c_int), ("node", ctypes.c_int), ("worker", ctypes.c_int),
                ("bytes", ctypes.c_uint64)]


_lib = None
_vp = ctypes.c_void_p
_i64 = ctypes.c_int64
_u64 = ctypes.c_uint64
_int = ctypes.c_int
_pint = ctypes.POINTER(ctypes.c_int)

_SIGS = {
    "northup_tree_create": [_vp],
    "northup_tree_add_node": [_vp, _int, _int, _int, _u64, _int, _pint],
    "northup_tree_set_block": [_vp, _int, _i64, _i64, _i64],
    "northup_tree_set_arena": [_vp, _int, _vp, _u64],
    "northup_tree_set_replica": [_vp, _int, _vp, _u64],
    "northup_tree_finalize": [_vp],
    "northup_tree_destroy": [_vp],
    "northup_fetch_node_type": [_vp, _int, _pint],
    "northup_get_parent": [_vp, _int, _pint],
    "northup_get_children_list": [_vp, _int, _pint, _int, _pint],
    "northup_get_level": [_vp, _int, _pint],
    "northup_get_max_treelevel": [_vp, _pint],
    "northup_get_num_nodes": [_vp, _pint],
    "northup_get_node_info": [_vp, _int, ctypes.POINTER(NodeInfo)],
    "northup_tree_print": [_vp, ctypes.c_char_p, ctypes.c_size_t, ctypes.POINTER(ctypes.c_size_t)],
    "northup_tree_link_info": [_vp, _vp, _vp, _vp],
    "northup_alloc": [_vp, _u64, _int, _vp],
    "northup_tree_set_file_dir": [_vp, ctypes.c_char_p],
    "northup_wrap_host": [_vp, _int, _vp, _u64, _vp],
    "northup_wrap_device": [_vp, _int, _vp, _u64, _vp],
    "northup_open_file": [_vp, _int, ctypes.c_char_p, _u64, _vp],
    "northup_buf_info": [_vp, _pint, ctypes.POINTER(_vp), ctypes.POINTER(_u64)],
    "northup_move_data": [_vp, _vp, _u64, _vp, _u64, _u64],
    "northup_move_data_down": [_vp, _vp, _vp, _u64, _u64, _int],
    "northup_move_data_up": [_vp, _vp, _vp, _u64, _u64],
    "northup_release": [_vp, _vp],
    "northup_gemm": [_vp, _vp, _vp, _vp, _i64, _i64, _i64],
    "northup_gemm_ex": [_vp, _vp, _vp, _vp, _i64, _i64, _i64, ctypes.POINTER(GemmOpts),
                        ctypes.POINTER(Stats)],
    "northup_leaf_gemm": [_vp, _i64, _vp, _i64, _vp, _i64, _i64, _i64, _i64, _int, _i64, _int, _vp],
    "northup_plan_create": [_vp, _i64, _i64, _i64, ctypes.POINTER(GemmOpts), _vp],
    "northup_plan_num_ops": [_vp, ctypes.POINTER(_i64)],
    "northup_plan_get_op": [_vp, _i64, ctypes.POINTER(Op)],
    "northup_plan_num_bufs": [_vp, _pint],
    "northup_plan_get_buf": [_vp, _int, ctypes.POINTER(PlanBuf)],
    "northup_plan_stats": [_vp, ctypes.POINTER(Stats)],
    "northup_plan_destroy": [_vp],
    "northup_partition": [_int, _i64, _i64, _i64, _pint, _pint],
    "northup_partition_region": [_int, _i64, _i64, _i64, _int, ctypes.POINTER(_i64),
                                 ctypes.POINTER(_i64), ctypes.POINTER(_i64), ctypes.POINTER(_i64)],
    "northup_file_tile_kpanels": [ctypes.c_char_p, ctypes.c_char_p, _i64, _i64, _i64],
    "northup_tree_set_local": [_vp, _int],
    "northup_peer_export": [_vp, _i64, _i64, _i64, ctypes.POINTER(GemmOpts), _vp, _u64,
                            ctypes.POINTER(_u64)],
    "northup_peer_import": [_vp, _int, _vp, _u64],
    "northup_hotspot_default_coeffs": [_i64, _i64, ctypes.POINTER(HotspotCoeffs)],
    "northup_hotspot_leaf": [_vp, _i64, _vp, _i64, _vp, _i64, _i64, _i64, _i64, _i64, _i64, _i64,
                             _int, ctypes.POINTER(HotspotCoeffs), _vp],
    "northup_hotspot": [_vp, _vp, _vp, _vp, _i64, _i64, _i64, ctypes.POINTER(HotspotCoeffs),
                        ctypes.POINTER(HotspotOpts), ctypes.POINTER(Stats)],
    "northup_hotspot_plan": [_vp, _i64, _i64, _i64, ctypes.POINTER(HotspotOpts), _vp],
    "northup_version": [],
    "northup_device_count": [],
}


def lib() -> ctypes.CDLL:
    """Load libnorthup.so (built by __graft_entry__.build()); raise if absent."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise NorthupError(NU_ESTATE, f"{LIB_PATH} is missing: run __graft_entry__.build() "
                                          "(there is no CPU fallback)")
        L = ctypes.CDLL(LIB_PATH)
        for name, args in _SIGS.items():
            f = getattr(L, name)
            f.argtypes = args
            f.restype = ctypes.c_int
        L.northup_last_error.argtypes = []
        L.northup_last_error.restype = ctypes.c_char_p
        _lib = L
    return _lib


def last_io_errno() -> int:
    """northup_last_io_errno: errno of the last failed file I/O (0: end of file)."""
    f = lib().northup_last_io_errno
    f.argtypes = []
    f.restype = ctypes.c_int
    return int(f())


def last_error() -> str:
    return lib().northup_last_error().decode(errors="replace")


def check(rc: int) -> int:
    if rc != NU_OK:
        raise NorthupError(rc, last_error())
    return rc


def header_symbols(path: str = HEADER) -> list[str]:
    """Function names declared in include/northup.h."""
    txt = open(path).read()
    return sorted(set(re.findall(r"^\s*(?:const\s+char\s*\*|int)\s+(northup_\w+)\s*\(", txt, re.M)))


def version() -> int:
    return lib().northup_version()


def device_count() -> int:
    return lib().northup_device_count()


def _stream_ptr(stream) -> int | None:
    if stream is None:
        return None
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream  # torch.cuda.Stream


def northup_leaf_gemm(A: int, lda: int, B: int, ldb: int, C: int, ldc: int, M: int, N: int,
                      K: int, accumulate: int = 0, k_chunk: int = 0, npass: int = 0,
                      stream=None) -> None:
    """Raw leaf call on device pointers (asynchronous on `stream`)."""
    check(lib().northup_leaf_gemm(A, lda, B, ldb, C, ldc, M, N, K, accumulate, k_chunk, npass,
                                  _stream_ptr(stream)))


def leaf_gemm(A, B, C, accumulate: bool = False, k_chunk: int = 0, npass: int = 0,
              stream=None) -> None:
    """C (+)= A @ B for row-major fp32 CUDA tensors (views with unit column stride)."""
    M, K = A.shape
    K2, N = B.shape
    if K2 != K or tuple(C.shape) != (M, N):
        raise NorthupError(NU_EINVAL, "shape mismatch")
    for t in (A, B, C):
        if not t.is_cuda or t.dtype.itemsize != 4 or (t.numel() and t.stride(1) != 1):
            raise NorthupError(NU_EINVAL, "row-major fp32 CUDA tensors required")
    if stream is None:
        import torch
        stream = torch.cuda.current_stream(A.device)
    northup_leaf_gemm(A.data_ptr(), A.stride(0) if M else K, B.data_ptr(), B.stride(0) if K else N,
                      C.data_ptr(), C.stride(0) if M else N, M, N, K, int(accumulate), k_chunk,
                      npass, stream)


def hotspot_coeffs(rows: int, cols: int) -> HotspotCoeffs:
    """northup_hotspot_default_coeffs (RH1/RH2), fp32."""
    k = HotspotCoeffs()
    check(lib().northup_hotspot_default_coeffs(rows, cols, ctypes.byref(k)))
    return k


def hotspot_opts(block: int = 0, halo: int = 0, leaf_iters: int = 0,
                 collect_timing: bool = False) -> HotspotOpts:
    o = HotspotOpts()
    o.block, o.halo, o.leaf_iters, o.collect_timing = block, halo, leaf_iters, int(collect_timing)
    return o


def hotspot_leaf(tin, pw, tout, iters: int, gy0: int = 0, gx0: int = 0, rows: int | None = None,
                 cols: int | None = None, coeffs: HotspotCoeffs | None = None, stream=None) -> None:
    """The HotSpot-2D leaf on window-shaped fp32 CUDA tensors (row-major views)."""
    wm, wn = tin.shape
    rows = wm if rows is None else rows
    cols = wn if cols is None else cols
    for x in (tin, pw, tout):
        if not x.is_cuda or x.dtype.itemsize != 4 or tuple(x.shape) != (wm, wn) or (x.numel() and x.stride(1) != 1):
            raise NorthupError(NU_EINVAL, "window-shaped row-major fp32 CUDA tensors required")
    if stream is None:
        import torch
        stream = torch.cuda.current_stream(tin.device)
    check(lib().northup_hotspot_leaf(tin.data_ptr(), tin.stride(0), pw.data_ptr(), pw.stride(0),
                                     tout.data_ptr(), tout.stride(0), wm, wn, gy0, gx0, rows, cols,
                                     iters, ctypes.byref(coeffs) if coeffs else None,
                                     _stream_ptr(stream)))


def file_tile_kpanels(src: str, dst: str, M: int, K: int, panel_k: int) -> None:
    """R15 preprocessing: row-major A file -> K-panel-major file."""
    check(lib().northup_file_tile_kpanels(src.encode(), dst.encode(), M, K, panel_k))


def partition(G: int, M: int, N: int, K: int = 0) -> tuple[int, int]:
    pr, pc = ctypes.c_int(), ctypes.c_int()
    check(lib().northup_partition(G, M, N, K, ctypes.byref(pr), ctypes.byref(pc)))
    return pr.value, pc.value


def partition_region(G: int, M: int, N: int, K: int, r: int) -> tuple[int, int, int, int]:
    v = [ctypes.c_int64() for _ in range(4)]
    check(lib().northup_partition_region(G, M, N, K, r, *[ctypes.byref(x) for x in v]))
    return tuple(x.value for x in v)


def make_opts(schedule: int = NU_SCHED_AUTO, k_chunk: int = 0, npass: int = 0,
              collect_timing: bool = False, replicate_result: bool = False,
              a_panel_k: int = 0, graph: bool = False, shared_staging: int = 0,
              queue_tiles: int = 0) -> GemmOpts:
    """northup_gemm_opts; shared_staging: 0 = auto (on for G > 1 uniform regions), -1 = off."""
    o = GemmOpts()
    o.queue_tiles = queue_tiles
    o.shared_staging = shared_staging
    o.a_panel_k = a_panel_k
    o.graph = int(graph)
    o.schedule = schedule
    o.k_chunk = k_chunk
    o.npass = npass
    o.collect_timing = int(collect_timing)
    o.replicate_result = int(replicate_result)
    return o


class Buf:
    """A northup_buf_t handle (owned by its tree)."""

    def __init__(self, tree: "Tree", handle: int):
        self.tree = tree
        self.handle = handle

    def info(self) -> tuple[int, int, int]:
        node, ptr, nbytes = ctypes.c_int(), ctypes.c_void_p(), ctypes.c_uint64()
        check(lib().northup_buf_info(self.handle, ctypes.byref(node), ctypes.byref(ptr),
                                     ctypes.byref(nbytes)))
        return node.value, ptr.value or 0, nbytes.value

    @property
    def ptr(self) -> int:
        return self.info()[1]

    def release(self) -> None:
        if self.handle:
            check(lib().northup_release(self.tree.handle, self.handle))
            self.handle = None


class Plan:
    """Host-only plan introspection (northup_plan_*)."""

    def __init__(self, tree: "Tree", M: int, N: int, K: int, opts=None, hotspot: bool = False):
        h = ctypes.c_void_p()
        create = lib().northup_hotspot_plan if hotspot else lib().northup_plan_create
        check(create(tree.handle, M, N, K, ctypes.byref(opts) if opts else None, ctypes.byref(h)))
        self.handle = h.value

    def ops(self) -> list[dict]:
        n = ctypes.c_int64()
        check(lib().northup_plan_num_ops(self.handle, ctypes.byref(n)))
        out = []
        for i in range(n.value):
            op = Op()
            check(lib().northup_plan_get_op(self.handle, i, ctypes.byref(op)))
            out.append(op.as_dict())
        return out

    def bufs(self) -> list[dict]:
        n = ctypes.c_int()
        check(lib().northup_plan_num_bufs(self.handle, ctypes.byref(n)))
        out = []
        for i in range(n.value):
            b = PlanBuf()
            check(lib().northup_plan_get_buf(self.handle, i, ctypes.byref(b)))
            out.append({k: getattr(b, k) for k, _ in b._fields_})
        return out

    def stats(self) -> dict:
        s = Stats()
        check(lib().northup_plan_stats(self.handle, ctypes.byref(s)))
        return s.as_dict()

    def close(self) -> None:
        if self.handle:
            lib().northup_plan_destroy(self.handle)
            self.handle = None

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass


class Tree:
    """northup_tree_t: build, finalize, allocate, move, multiply."""

    def __init__(self):
        h = ctypes.c_void_p()
        check(lib().northup_tree_create(ctypes.byref(h)))
        self.handle = h.value
        self._keep = []   # python objects whose memory the tree references

    # -- construction (Listing 1)
    def add_node(self, parent: int, storage: int, physical_id: int = -1, capacity: int = 0,
                 processor: int = NU_PROC_NONE) -> int:
        nid = ctypes.c_int()
        check(lib().northup_tree_add_node(self.handle, parent, storage, physical_id, capacity,
                                          processor, ctypes.byref(nid)))
        return nid.value

    def set_block(self, node: int, bm: int, bn: int, bk: int) -> None:
        check(lib().northup_tree_set_block(self.handle, node, bm, bn, bk))

    def set_arena(self, node: int, ptr: int, nbytes: int, keepalive=None) -> None:
        check(lib().northup_tree_set_arena(self.handle, node, ptr, nbytes))
        if keepalive is not None:
            self._keep.append(keepalive)

    def set_replica(self, node: int, ptr: int, nbytes: int, keepalive=None) -> None:
        check(lib().northup_tree_set_replica(self.handle, node, ptr, nbytes))
        if keepalive is not None:
            self._keep.append(keepalive)

    def set_file_dir(self, d: str) -> None:
        check(lib().northup_tree_set_file_dir(self.handle, d.encode()))

    def link_info(self) -> dict:
        """northup_tree_link_info: what finalize measured (PCIe, P2P, NUMA binding)."""
        g, p, n = ctypes.c_double(), ctypes.c_int(), ctypes.c_int()
        check(lib().northup_tree_link_info(self.handle, ctypes.byref(g), ctypes.byref(p), ctypes.byref(n)))
        return {"pcie_gbs": g.value, "p2p_ok": bool(p.value), "numa_bound_workers": n.value}

    def finalize(self) -> None:
        check(lib().northup_tree_finalize(self.handle))

    # -- multi-process siblings (one process per GPU)
    def set_local(self, node: int) -> None:
        """This process runs only HBM node `node` (before finalize)."""
        check(lib().northup_tree_set_local(self.handle, node))

    def peer_export(self, M: int, N: int, K: int, opts: GemmOpts | None = None) -> bytes:
        """Plan the GEMM, allocate the local arena; CUDA IPC handles for the peers."""
        n = ctypes.c_uint64()
        o = ctypes.byref(opts) if opts else None
        lib().northup_peer_export(self.handle, M, N, K, o, None, 0, ctypes.byref(n))
        buf = ctypes.create_string_buffer(n.value)
        check(lib().northup_peer_export(self.handle, M, N, K, o, buf, n.value, ctypes.byref(n)))
        return buf.raw[: n.value]

    def peer_import(self, worker: int, blob: bytes) -> None:
        check(lib().northup_peer_import(self.handle, worker, blob, len(blob)))

    def destroy(self) -> None:
        if self.handle:
            check(lib().northup_tree_destroy(self.handle))
            self.handle = None
            self._keep = []

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.destroy()

    def __del__(self):
        try:
            self.destroy()
        except Exception:
            pass

    # -- queries
    def fetch_node_type(self, node: int) -> int:
        v = ctypes.c_int()
        check(lib().northup_fetch_node_type(self.handle, node, ctypes.byref(v)))
        return v.value

    def get_parent(self, node: int) -> int:
        v = ctypes.c_int()
        check(lib().northup_get_parent(self.handle, node, ctypes.byref(v)))
        return v.value

    def get_children_list(self, node: int) -> list[int]:
        n = ctypes.c_int()
        check(lib().northup_get_children_list(self.handle, node, None, 0, ctypes.byref(n)))
        arr = (ctypes.c_int * max(1, n.value))()
        check(lib().northup_get_children_list(self.handle, node, arr, n.value, ctypes.byref(n)))
        return list(arr)[: n.value]

    def get_level(self, node: int) -> int:
        v = ctypes.c_int()
        check(lib().northup_get_level(self.handle, node, ctypes.byref(v)))
        return v.value

    def get_max_treelevel(self) -> int:
        v = ctypes.c_int()
        check(lib().northup_get_max_treelevel(self.handle, ctypes.byref(v)))
        return v.value

    def num_nodes(self) -> int:
        v = ctypes.c_int()
        check(lib().northup_get_num_nodes(self.handle, ctypes.byref(v)))
        return v.value

    def node_info(self, node: int) -> dict:
        info = NodeInfo()
        check(lib().northup_get_node_info(self.handle, node, ctypes.byref(info)))
        return {k: getattr(info, k) for k, _ in info._fields_}

    def print(self) -> str:
        need = ctypes.c_size_t()
        check(lib().northup_tree_print(self.handle, None, 0, ctypes.byref(need)))
        buf = ctypes.create_string_buffer(need.value)
        check(lib().northup_tree_print(self.handle, buf, need.value, None))
        return buf.value.decode()

    # -- unified data API (Table I)
    def alloc(self, nbytes: int, node: int) -> Buf:
        h = ctypes.c_void_p()
        check(lib().northup_alloc(self.handle, nbytes, node, ctypes.byref(h)))
        return Buf(self, h.value)

    def wrap_host(self, node: int, ptr: int, nbytes: int, keepalive=None) -> Buf:
        h = ctypes.c_void_p()
        check(lib().northup_wrap_host(self.handle, node, ptr, nbytes, ctypes.byref(h)))
        if keepalive is not None:
            self._keep.append(keepalive)
        return Buf(self, h.value)

    def wrap_device(self, node: int, ptr: int, nbytes: int, keepalive=None) -> Buf:
        h = ctypes.c_void_p()
        check(lib().northup_wrap_device(self.handle, node, ptr, nbytes, ctypes.byref(h)))
        if keepalive is not None:
            self._keep.append(keepalive)
        return Buf(self, h.value)

    def open_file(self, node: int, path: str, nbytes: int) -> Buf:
        h = ctypes.c_void_p()
        check(lib().northup_open_file(self.handle, node, path.encode(), nbytes, ctypes.byref(h)))
        return Buf(self, h.value)

    def move_data(self, dst: Buf, dst_off: int, src: Buf, src_off: int, nbytes: int) -> None:
        check(lib().northup_move_data(self.handle, dst.handle, dst_off, src.handle, src_off, nbytes))

    def move_data_down(self, dst: Buf, src: Buf, nbytes: int, src_off: int, child: int) -> None:
        check(lib().northup_move_data_down(self.handle, dst.handle, src.handle, nbytes, src_off, child))

    def move_data_up(self, dst: Buf, src: Buf, nbytes: int, dst_off: int) -> None:
        check(lib().northup_move_data_up(self.handle, dst.handle, src.handle, nbytes, dst_off))

    def release(self, b: Buf) -> None:
        b.release()

    # -- the GEMM (§IV-A)
    def gemm(self, A: Buf, B: Buf, C: Buf, M: int, N: int, K: int,
             opts: GemmOpts | None = None) -> dict:
        st = Stats()
        check(lib().northup_gemm_ex(self.handle, A.handle, B.handle, C.handle, M, N, K,
                                    ctypes.byref(opts) if opts else None, ctypes.byref(st)))
        return st.as_dict()

    def plan(self, M: int, N: int, K: int, opts: GemmOpts | None = None) -> Plan:
        return Plan(self, M, N, K, opts)

    # -- HotSpot-2D (NEXT-3)
    def hotspot(self, T: Buf, P: Buf, Tout: Buf, rows: int, cols: int, iters: int,
                opts: HotspotOpts | None = None, coeffs: HotspotCoeffs | None = None) -> dict:
        st = Stats()
        check(lib().northup_hotspot(self.handle, T.handle, P.handle, Tout.handle, rows, cols, iters,
                                    ctypes.byref(coeffs) if coeffs else None,
                                    ctypes.byref(opts) if opts else None, ctypes.byref(st)))
        return st.as_dict()

    def hotspot_plan(self, rows: int, cols: int, iters: int, opts: HotspotOpts | None = None) -> "Plan":
        return Plan(self, rows, cols, iters, opts, hotspot=True)


def host_tree(num_gpus: int = 1, hbm_capacity: int = 0, smem_leaf: bool = True,
              devices=None) -> tuple[Tree, list[int]]:
    """HOST root -> num_gpus x HBM (-> SMEM/TMEM leaf).  Returns (tree, hbm ids)."""
    t = Tree()
    root = t.add_node(-1, NU_HOST)
    hbm = []
    for g in range(num_gpus):
        dev = devices[g] if devices is not None else g
        if smem_leaf:
            h = t.add_node(root, NU_HBM, dev, hbm_capacity)
            t.add_node(h, NU_SMEM, dev, 227 * 1024, NU_PROC_SM100)
        else:
            h = t.add_node(root, NU_HBM, dev, hbm_capacity, NU_PROC_SM100)
        hbm.append(h)
    return t, hbm


def hbm_tree(device: int = 0, smem_leaf: bool = True) -> Tree:
    """Single-GPU in-HBM tree (CS4): HBM root (-> SMEM/TMEM leaf)."""
    t = Tree()
    if smem_leaf:
        h = t.add_node(-1, NU_HBM, device)
        t.add_node(h, NU_SMEM, device, 227 * 1024, NU_PROC_SM100)
    else:
        t.add_node(-1, NU_HBM, device, 0, NU_PROC_SM100)
    return t
