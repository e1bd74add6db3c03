"""B200-native ADDS single-source shortest paths (PPoPP'21 hot path).

Thin ctypes binding over ``libsssp.so`` (``include/sssp.h``): argument
marshalling only -- every step of the SSSP runs in the sm_100a kernels under
``csrc/``.  There is no CPU fallback: if the extension is not built, or no
sm_100 device is present, calls raise.

PyTorch is used for device memory (output tensors) and streams only.

    >>> import paper_conf_ppopp_wangfl21_b200 as sssp
    >>> g = sssp.Graph(row_offsets, col, w)          # numpy / torch (host or cuda)
    >>> d = g.run(source)                            # torch.int64 [n] on cuda (UINT64_MAX -> -1)
    >>> D = g.run_batch(sources)                     # torch.int64 [k, n]
    >>> g.stats()                                    # dict (work counts, Delta, timings)
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

from . import _build

LIB_PATH = _build.LIB
_libs = {}

INF = 0xFFFFFFFFFFFFFFFF

SSSP_FLAG_TRACE = 0x1
SSSP_FLAG_ASYNC = 0x2
SSSP_FLAG_NO_RETRY = 0x4
SSSP_FLAG_NO_LOCAL = 0x8
SSSP_FLAG_PROFILE = 0x10
SSSP_FLAG_L2_PERSIST = 0x20
SSSP_FLAG_ADAPT_ACTIVE = 0x40  # (default since round 2)
SSSP_FLAG_FIXED_ACTIVE = 0x1000
SSSP_FLAG_CHUNKED_RING = 0x2000
SSSP_FLAG_WIDE_ROWS = 0x4000
SSSP_FLAG_NO_WARP_LOCAL = 0x80
SSSP_FLAG_WARP_LOCAL = 0x100
SSSP_FLAG_FILTER16 = 0x200
SSSP_FLAG_RELABEL = 0x400
SSSP_FLAG_NO_RELABEL = 0x800
SSSP_WORKER_AUTO = 0
SSSP_WORKER_CTA = 1
PROFILE_FIELDS = ["cyc_claim", "cyc_idle", "cyc_pop", "cyc_scan", "cyc_rounds", "cyc_flush", "cyc_complete",
                  "cyc_total", "n_ring_batches", "n_local_batches", "n_idle", "n_flush", "n_rounds", "n_ctas",
                  "cyc_window", "n_windows"]
SSSP_ALGO_ADDS = 0
SSSP_ALGO_NEAR_FAR = 1
SSSP_DELTA_H_RING_SPAN = 0
SSSP_DELTA_H_NEARFAR = 1
SSSP_DELTA_H_MAXW_OVER_D = 2
SSSP_DELTA_DYNAMIC = 0
SSSP_DELTA_STATIC = 1

STATUS = {
    0: "SSSP_OK", 1: "SSSP_ERR_INVALID_ARGUMENT", 2: "SSSP_ERR_INVALID_GRAPH", 3: "SSSP_ERR_OUT_OF_MEMORY",
    4: "SSSP_ERR_CUDA", 5: "SSSP_ERR_WORKLIST_OVERFLOW", 6: "SSSP_ERR_TIMEOUT", 7: "SSSP_ERR_DEVICE_MISMATCH",
    8: "SSSP_ERR_BUSY", 9: "SSSP_ERR_NO_DEVICE",
}


class SSSPError(RuntimeError):
    def __init__(self, status: int, detail: str):
        super().__init__(f"{STATUS.get(status, status)}: {detail}")
        self.status = status
        self.detail = detail


class sssp_options(ctypes.Structure):
    _fields_ = [
        ("struct_size", ctypes.c_uint32), ("device", ctypes.c_int32), ("num_buckets", ctypes.c_uint32),
        ("delta_mode", ctypes.c_uint32), ("delta_init", ctypes.c_uint64), ("clip_pct", ctypes.c_uint32),
        ("settle_head_switches", ctypes.c_uint32), ("util_lo_pct", ctypes.c_uint32),
        ("util_hi_pct", ctypes.c_uint32), ("waste_lo_permille", ctypes.c_uint32),
        ("waste_hi_permille", ctypes.c_uint32), ("period_us", ctypes.c_uint32),
        ("delta_heuristic", ctypes.c_uint32),
        ("dist_bits", ctypes.c_uint32), ("ring_items", ctypes.c_uint64),
        ("flags", ctypes.c_uint32), ("block_threads", ctypes.c_uint32), ("grid_ctas", ctypes.c_uint32),
        ("batch_min", ctypes.c_uint32), ("timeout_ms", ctypes.c_uint32), ("trace_capacity", ctypes.c_uint32),
        ("active_init", ctypes.c_uint32), ("local_max", ctypes.c_uint32), ("max_backoff_ns", ctypes.c_uint32),
        ("startup_permille", ctypes.c_uint32), ("concurrent_sources", ctypes.c_uint32),
        ("algorithm", ctypes.c_uint32), ("split_degree", ctypes.c_uint32), ("worker", ctypes.c_uint32), ("reserved2", ctypes.c_uint32 * 1),
    ]


class sssp_stats(ctypes.Structure):
    _fields_ = [
        ("vertices_processed", ctypes.c_uint64), ("edges_relaxed", ctypes.c_uint64), ("pushes", ctypes.c_uint64),
        ("stale_skips", ctypes.c_uint64), ("reachable", ctypes.c_uint64), ("reach_edges", ctypes.c_uint64),
        ("max_dist", ctypes.c_uint64), ("init_delta_log2", ctypes.c_uint32), ("final_delta_log2", ctypes.c_uint32),
        ("head_switches", ctypes.c_uint32), ("delta_changes", ctypes.c_uint32), ("retries", ctypes.c_uint32),
        ("dist_bits", ctypes.c_uint32), ("grid_ctas", ctypes.c_uint32), ("block_threads", ctypes.c_uint32),
        ("runs", ctypes.c_uint32), ("trace_entries", ctypes.c_uint32), ("kernel_ms", ctypes.c_float),
        ("total_ms", ctypes.c_float), ("status", ctypes.c_uint32), ("batch_ms", ctypes.c_float),
        ("concurrency", ctypes.c_uint32), ("worker", ctypes.c_uint32), ("ring_bytes", ctypes.c_uint64),
    ]


class sssp_trace_entry(ctypes.Structure):
    _fields_ = [
        ("time_ns", ctypes.c_uint64), ("head", ctypes.c_uint64), ("pending_total", ctypes.c_uint64),
        ("pending_window", ctypes.c_uint64), ("pending_tail", ctypes.c_uint64), ("delta_log2", ctypes.c_uint32),
        ("active", ctypes.c_uint32), ("waste_permille", ctypes.c_uint32), ("reason", ctypes.c_uint32),
    ]


class sssp_certificate(ctypes.Structure):
    _fields_ = [
        ("exact", ctypes.c_uint32), ("source_ok", ctypes.c_uint32), ("violated_arcs", ctypes.c_uint64),
        ("first_violated_tail", ctypes.c_uint64), ("unanchored", ctypes.c_uint64),
        ("first_unanchored", ctypes.c_uint64), ("bad_markers", ctypes.c_uint64), ("reachable", ctypes.c_uint64),
        ("reach_edges", ctypes.c_uint64), ("fixpoint_rounds", ctypes.c_uint32), ("reserved", ctypes.c_uint32),
    ]


# (name, restype, argtypes) for every symbol declared in include/sssp.h
_P = ctypes.c_void_p
SIGNATURES = [
    ("sssp_options_default", None, [ctypes.POINTER(sssp_options)]),
    ("sssp_graph_create", ctypes.c_int,
     [ctypes.c_uint32, ctypes.c_uint64, _P, _P, _P, ctypes.POINTER(sssp_options), ctypes.POINTER(_P)]),
    ("sssp_graph_create_f32", ctypes.c_int,
     [ctypes.c_uint32, ctypes.c_uint64, _P, _P, _P, ctypes.POINTER(sssp_options), ctypes.POINTER(_P)]),
    ("sssp_graph_destroy", ctypes.c_int, [_P]),
    ("sssp_set_options", ctypes.c_int, [_P, ctypes.POINTER(sssp_options)]),
    ("sssp_run", ctypes.c_int, [_P, ctypes.c_uint32, _P, _P]),
    ("sssp_run_batch", ctypes.c_int, [_P, _P, ctypes.c_uint32, _P, _P]),
    ("sssp_run_f32", ctypes.c_int, [_P, ctypes.c_uint32, _P, _P]),
    ("sssp_run_batch_f32", ctypes.c_int, [_P, _P, ctypes.c_uint32, _P, _P]),
    ("sssp_get_stats", ctypes.c_int, [_P, ctypes.POINTER(sssp_stats)]),
    ("sssp_get_trace", ctypes.c_int, [_P, _P, ctypes.c_uint32, ctypes.POINTER(ctypes.c_uint32)]),
    ("sssp_get_profile", ctypes.c_int, [_P, _P, ctypes.c_uint32, ctypes.POINTER(ctypes.c_uint32)]),
    ("sssp_certify", ctypes.c_int, [_P, ctypes.c_uint32, _P, ctypes.POINTER(sssp_certificate), _P]),
    ("sssp_graph_info", ctypes.c_int, [_P, _P, _P, _P, _P, _P]),
    ("sssp_graph_layout", ctypes.c_int, [_P, _P, _P]),
    ("sssp_bucket_offset", ctypes.c_uint32, [ctypes.c_uint64, ctypes.c_uint32, ctypes.c_uint64, ctypes.c_uint32]),
    ("sssp_status_string", ctypes.c_char_p, [ctypes.c_int]),
    ("sssp_last_error", ctypes.c_char_p, []),
    ("sssp_version", ctypes.c_char_p, []),
]


def lib(variant: str = ""):
    """Load libsssp.so (raises if it was not built: there is no fallback).

    variant "fuzz" loads libsssp_fuzz.so: the same library built with -DSSSP_FUZZ,
    which injects hash-driven delays at the worklist's reserve / publish / claim /
    complete / head-CAS points (schedule fuzzing for the parity tests)."""
    L = _libs.get(variant)
    if L is None:
        path = _build.variant_path(variant)
        if not os.path.exists(path):
            raise RuntimeError(f"{path} is missing: build the CUDA extension first "
                               "(python -c 'import __graft_entry__ as g; g.build()')")
        L = ctypes.CDLL(path)
        for name, res, args in SIGNATURES:
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _libs[variant] = L
    return L


def _check(st: int, L=None):
    if st != 0:
        raise SSSPError(st, (L or lib()).sssp_last_error().decode())


# ------------------------------------------------------------------ same-name C wrappers
def sssp_options_default(**overrides) -> sssp_options:
    o = sssp_options()
    lib().sssp_options_default(ctypes.byref(o))
    for k, v in overrides.items():
        if not hasattr(o, k):
            raise KeyError(k)
        setattr(o, k, v)
    return o


def sssp_bucket_offset(d: int, delta_log2: int, head: int, num_buckets: int = 32) -> int:
    return int(lib().sssp_bucket_offset(d, delta_log2, head, num_buckets))


def sssp_status_string(st: int) -> str:
    return lib().sssp_status_string(st).decode()


def sssp_version() -> str:
    return lib().sssp_version().decode()


def _torch():
    try:
        import torch
        return torch
    except ImportError:  # pragma: no cover
        return None


def _as_host_or_dev(a, dtype, what: str):
    """Return (pointer, keepalive) for a numpy array or a torch tensor (host or cuda)
    holding ``dtype`` values (np.uint64 / np.uint32 / np.float32).

    Same-width integer types are passed through (their bits are the values the ABI
    reads); other integer types are range-checked and converted; anything else
    (e.g. float64 weights, int64 column indices beyond 2^32) raises instead of
    being reinterpreted."""
    torch = _torch()
    want = np.dtype(dtype)
    if torch is not None and isinstance(a, torch.Tensor):
        t = a.contiguous()
        if want.kind == "f":
            if t.dtype != torch.float32:
                raise TypeError(f"{what}: float32 expected, got {t.dtype}")
            return t.data_ptr(), t
        if t.dtype.is_floating_point or t.dtype.is_complex or t.dtype == torch.bool:
            raise TypeError(f"{what}: integer tensor expected, got {t.dtype}")
        if t.element_size() == want.itemsize:
            if t.numel() and t.dtype.is_signed and int(t.min()) < 0:
                raise ValueError(f"{what}: negative values")
            return t.data_ptr(), t
        if t.numel() and (int(t.min()) < 0 or int(t.max()) >= (1 << (8 * want.itemsize))):
            raise ValueError(f"{what}: values out of range for {want}")
        t = t.to(torch.int64 if want.itemsize == 8 else torch.int32).contiguous()
        return t.data_ptr(), t
    arr = np.asarray(a)
    if arr.dtype != want:
        if want.kind == "f":
            raise TypeError(f"{what}: float32 expected, got {arr.dtype}")
        if arr.dtype.kind not in "iu":
            raise TypeError(f"{what}: integer array expected, got {arr.dtype}")
        if arr.size and (int(arr.min()) < 0 or int(arr.max()) >= (1 << (8 * want.itemsize))):
            raise ValueError(f"{what}: values out of range for {want}")
    arr = np.ascontiguousarray(arr, dtype=want)
    return arr.ctypes.data, arr


def _is_float(a) -> bool:
    torch = _torch()
    if torch is not None and isinstance(a, torch.Tensor):
        return a.dtype.is_floating_point
    return np.asarray(a).dtype.kind == "f"


def _check_out(out, f32: bool, numel: int, device: int):
    """The ABI writes numel 8-byte (4-byte float) values: refuse anything else."""
    torch = _torch()
    if f32 and out.dtype != torch.float32:
        raise TypeError(f"out: float32 expected for a float32-weight graph, got {out.dtype}")
    if not f32 and out.dtype not in (torch.int64, getattr(torch, "uint64", torch.int64)):
        raise TypeError(f"out: int64 expected, got {out.dtype}")
    if not out.is_contiguous():
        raise ValueError("out must be contiguous")
    if out.numel() != numel:
        raise ValueError(f"out has {out.numel()} elements, {numel} expected")
    if out.is_cuda and out.device.index != device:
        raise ValueError(f"out is on {out.device}, the graph on cuda:{device}")


def _stream_ptr(stream):
    if stream is None:
        import torch
        return torch.cuda.current_stream().cuda_stream
    if isinstance(stream, int):
        return stream
    return stream.cuda_stream


class Graph:
    """A CSR graph resident on one GPU plus its ADDS workspace (``sssp_graph*``)."""

    def __init__(self, row_offsets, col, w, options: sssp_options | None = None, device: int = 0,
                 variant: str = "", **opt):
        self._L = L = lib(variant)
        self._h = _P()
        if options is None:
            options = sssp_options_default(device=device, **opt)
        self.options = options
        self.n = int(len(row_offsets) - 1)
        self.m = int(len(col))
        self.f32 = _is_float(w)
        po, k1 = _as_host_or_dev(row_offsets, np.uint64, "row_offsets")
        pc, k2 = _as_host_or_dev(col, np.uint32, "col")
        pw, k3 = _as_host_or_dev(w, np.float32 if self.f32 else np.uint32, "w")
        create = L.sssp_graph_create_f32 if self.f32 else L.sssp_graph_create
        _check(create(self.n, self.m, po, pc, pw, ctypes.byref(options), ctypes.byref(self._h)), L)
        self.device = options.device

    @classmethod
    def from_csr(cls, csr, weights=None, **kw):
        """``weights`` overrides csr.w (e.g. float32 weights from graphgen.float_weights)."""
        return cls(csr.row_offsets, csr.col, csr.w if weights is None else weights, **kw)

    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            self._L.sssp_graph_destroy(self._h)
            self._h = _P()

    __del__ = close

    def __enter__(self):
        return self

    def __exit__(self, *exc):
        self.close()

    def set_options(self, **overrides):
        o = sssp_options()
        ctypes.memmove(ctypes.byref(o), ctypes.byref(self.options), ctypes.sizeof(o))
        for k, v in overrides.items():
            setattr(o, k, v)
        _check(self._L.sssp_set_options(self._h, ctypes.byref(o)), self._L)
        self.options = o

    def run(self, source: int, out=None, stream=None):
        """dist[v] from ``source`` as a cuda tensor: torch.int64 (UINT64_MAX reads as -1) for
        integer weights, torch.float32 (+inf when unreachable) for float32 weights."""
        import torch
        if out is None:
            out = torch.empty(self.n, dtype=torch.float32 if self.f32 else torch.int64, device=f"cuda:{self.device}")
        _check_out(out, self.f32, self.n, self.device)
        fn = self._L.sssp_run_f32 if self.f32 else self._L.sssp_run
        _check(fn(self._h, int(source), out.data_ptr(), _stream_ptr(stream)), self._L)
        return out

    def run_host(self, source: int, out: np.ndarray | None = None, stream=None) -> np.ndarray:
        """Same, into host memory (the library copies the result back)."""
        if out is None:
            out = np.empty(self.n, dtype=np.float32 if self.f32 else np.uint64)
        if out.dtype != (np.float32 if self.f32 else np.uint64) or out.size != self.n or not out.flags.c_contiguous:
            raise ValueError("out: contiguous float32 (float graphs) / uint64 array of n entries expected")
        fn = self._L.sssp_run_f32 if self.f32 else self._L.sssp_run
        _check(fn(self._h, int(source), out.ctypes.data, _stream_ptr(stream)), self._L)
        return out

    def run_batch(self, sources, out=None, stream=None):
        """[k, n] torch.int64 distances for k sources (row i <-> sources[i])."""
        import torch
        src = np.ascontiguousarray(sources, dtype=np.uint32)
        if out is None:
            out = torch.empty((len(src), self.n), dtype=torch.float32 if self.f32 else torch.int64,
                              device=f"cuda:{self.device}")
        _check_out(out, self.f32, len(src) * self.n, self.device)
        fn = self._L.sssp_run_batch_f32 if self.f32 else self._L.sssp_run_batch
        _check(fn(self._h, src.ctypes.data, len(src), out.data_ptr(), _stream_ptr(stream)), self._L)
        return out

    def stats(self) -> dict:
        s = sssp_stats()
        _check(self._L.sssp_get_stats(self._h, ctypes.byref(s)), self._L)
        d = {f: getattr(s, f) for f, _ in sssp_stats._fields_ if f != "reserved"}
        return d

    def trace(self):
        cap = self.options.trace_capacity or 65536
        buf = (sssp_trace_entry * cap)()
        cnt = ctypes.c_uint32(0)
        _check(self._L.sssp_get_trace(self._h, buf, cap, ctypes.byref(cnt)), self._L)
        return [{f: getattr(buf[i], f) for f, _ in sssp_trace_entry._fields_} for i in range(cnt.value)]

    def profile(self) -> dict:
        buf = (ctypes.c_uint64 * 16)()
        cnt = ctypes.c_uint32(0)
        _check(self._L.sssp_get_profile(self._h, buf, 16, ctypes.byref(cnt)), self._L)
        return {k: int(buf[i]) for i, k in enumerate(PROFILE_FIELDS)}

    def certify(self, source: int, dist, stream=None) -> dict:
        """GPU certificate of a distance vector (sssp_certify): ``dist`` = torch tensor (device
        or host) or numpy array of n entries (int64/uint64, float32 for float graphs)."""
        torch = _torch()
        if torch is not None and isinstance(dist, torch.Tensor):
            t = dist.contiguous()
            if t.numel() != self.n or t.element_size() != (4 if self.f32 else 8):
                raise ValueError("dist: n entries of the graph's distance type expected")
            ptr, keep = t.data_ptr(), t
        else:
            keep = np.ascontiguousarray(dist, dtype=np.float32 if self.f32 else np.uint64)
            if keep.size != self.n:
                raise ValueError("dist: n entries expected")
            ptr = keep.ctypes.data
        c = sssp_certificate()
        _check(self._L.sssp_certify(self._h, int(source), ptr, ctypes.byref(c), _stream_ptr(stream)), self._L)
        del keep
        return {f: getattr(c, f) for f, _ in sssp_certificate._fields_ if f != "reserved"}

    def info(self) -> dict:
        n, m, sw, mw, hk = ctypes.c_uint32(), ctypes.c_uint64(), ctypes.c_uint64(), ctypes.c_uint32(), ctypes.c_uint32()
        _check(self._L.sssp_graph_info(self._h, ctypes.byref(n), ctypes.byref(m), ctypes.byref(sw), ctypes.byref(mw),
                                       ctypes.byref(hk)), self._L)
        rl, mi = ctypes.c_uint32(), ctypes.c_uint32()
        _check(self._L.sssp_graph_layout(self._h, ctypes.byref(rl), ctypes.byref(mi)), self._L)
        return {"n": n.value, "m": m.value, "sum_w": sw.value, "max_w": mw.value, "heuristic_delta_log2": hk.value,
                "relabeled": rl.value, "max_indeg": mi.value}


def to_u64(t) -> np.ndarray:
    """torch.int64 distances -> numpy uint64 (UINT64_MAX for unreachable)."""
    return t.detach().cpu().numpy().view(np.uint64)
