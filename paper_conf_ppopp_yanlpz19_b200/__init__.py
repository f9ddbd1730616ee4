"""Harmonia (PPoPP'19) batched B+tree search on B200 — Python binding of libharmonia.so.

Argument marshalling only: every step of build, search, range and update runs in the CUDA
kernels of ``csrc/`` behind the C ABI declared in ``include/harmonia.h``.  PyTorch provides
device memory (tensors), streams and, in ``dist``, process groups.  There is no CPU
fallback: if the shared library cannot be loaded the import of any entry point raises.
"""
from __future__ import annotations

import ctypes as C
import os

import numpy as np

from . import _build

__all__ = ["Tree", "HarmoniaError", "QueryOpts", "lib", "kernel_launches", "psa_bits_auto",
           "NOT_FOUND", "KEY_PAD", "route_partition", "scatter_results"]

NOT_FOUND = 0xFFFFFFFFFFFFFFFF
KEY_PAD = 0xFFFFFFFFFFFFFFFF
QF_NO_PS_SMEM = 1
QF_GATHER = 2
QF_LINEAR = 4
QF_PSA_GLOBAL = 8
QF_ILP1 = 16
QF_PSA_COARSE = 32
QF_SCATTER_RETURN = 256
QF_NO_L2_WINDOW = 4096
QF_PER_LANE = 1024
QF_RANGE_GROUP = 2048
QF_PSA_L16 = 8192
QF_PSA_L8 = 16384
QF_NO_RANGE_LANE = 32768
QF_HOST_UNORDERED = 65536
_STATUS = {0: "OK", 1: "INVALID_ARG", 2: "UNSORTED", 3: "RESERVED", 4: "OUT_OF_MEMORY", 5: "CUDA",
           6: "DEVICE_MISMATCH", 7: "TOO_LARGE"}


class HarmoniaError(RuntimeError):
    def __init__(self, status: int, what: str = ""):
        self.status = status
        msg = lib().harmonia_status_string(status).decode()
        if status == 5:
            msg += f" (cudaError {lib().harmonia_last_cuda_error()})"
        super().__init__(f"{what}: {_STATUS.get(status, status)}: {msg}")


class BuildOpts(C.Structure):
    _fields_ = [("fanout", C.c_uint32), ("fill", C.c_float), ("keys_on_device", C.c_int32),
                ("reserved", C.c_int32)]


class QueryOpts(C.Structure):
    _fields_ = [("group_size", C.c_int32), ("psa_bits", C.c_int32), ("smem_levels", C.c_int32),
                ("flags", C.c_int32), ("window", C.c_uint64), ("lane_queries", C.c_uint32),
                ("sort_chunk", C.c_uint32), ("l2_window_bytes", C.c_uint64)]


class PlanInfo(C.Structure):
    _fields_ = [("group_size", C.c_int32), ("psa_bits", C.c_int32), ("smem_levels", C.c_int32),
                ("ps_in_smem", C.c_int32), ("window", C.c_uint64), ("smem_bytes", C.c_uint32),
                ("smem_nodes", C.c_uint32), ("staged_return", C.c_uint32), ("lane_queries", C.c_uint32),
                ("warp_shared", C.c_uint32), ("sort_chunk", C.c_uint32),
                ("l2_window_bytes", C.c_uint64), ("psa_levels", C.c_uint32), ("chunk_group", C.c_uint32)]


class Info(C.Structure):
    _fields_ = [("n_keys", C.c_uint64), ("fanout", C.c_uint32), ("height", C.c_uint32),
                ("psa_bits_auto", C.c_uint32), ("group_size_auto", C.c_uint32),
                ("n_nodes", C.c_uint64), ("n_internal", C.c_uint64), ("n_leaves", C.c_uint64),
                ("level_start", C.c_uint64 * 65), ("key_region_bytes", C.c_uint64),
                ("ps_bytes", C.c_uint64), ("value_bytes", C.c_uint64), ("min_key", C.c_uint64),
                ("max_key", C.c_uint64), ("device", C.c_int32), ("reserved", C.c_int32)]


_lib = None
_vp = C.c_void_p
_u64 = C.c_uint64
_sz = C.c_size_t


def lib():
    """Load libharmonia.so (building it in-tree if it is missing).  Raises if unavailable."""
    global _lib
    if _lib is None:
        path = os.environ.get("HARMONIA_LIB") or _build.LIB  # HARMONIA_LIB: an alternative build (experiments)
        if path == _build.LIB and not os.path.exists(path):
            _build.build()
        L = C.CDLL(path)
        sig = {
            "harmonia_build": (C.c_int, [_vp, _vp, _u64, C.POINTER(BuildOpts), _vp, C.POINTER(_vp)]),
            "harmonia_destroy": (None, [_vp]),
            "harmonia_get_info": (C.c_int, [_vp, C.POINTER(Info)]),
            "harmonia_export_layout": (C.c_int, [_vp, _vp, _vp, _vp]),
            "harmonia_search_workspace_bytes": (_sz, [_vp, _u64, C.POINTER(QueryOpts)]),
            "harmonia_search_batch": (C.c_int, [_vp, _vp, _u64, _vp, _vp, _sz, C.POINTER(QueryOpts), _vp]),
            "harmonia_search_host_workspace_bytes": (_sz, [_vp, _u64, C.POINTER(QueryOpts)]),
            "harmonia_search_batch_host": (C.c_int, [_vp, _vp, _u64, _vp, _vp, _sz, C.POINTER(QueryOpts), _vp]),
            "harmonia_range_workspace_bytes": (_sz, [_vp, _u64, C.POINTER(QueryOpts)]),
            "harmonia_range_batch": (C.c_int, [_vp, _vp, _vp, _u64, C.c_uint32, _vp, _vp, _vp, _vp, _sz,
                                               C.POINTER(QueryOpts), _vp]),
            "harmonia_update_workspace_bytes": (_sz, [_vp, _u64]),
            "harmonia_update_batch": (C.c_int, [_vp, _vp, _vp, _vp, _u64, _vp, _sz, _vp]),
            "harmonia_update_batch_seq": (C.c_int, [_vp, _vp, _vp, _vp, _vp, _u64, _vp, _sz, _vp]),
            "harmonia_update_validate": (C.c_int, [_vp, _vp, _vp, _u64, _vp, _vp]),
            "harmonia_update_last_mode": (C.c_int, [_vp]),
            "harmonia_route_update_payload": (C.c_int, [_vp, _vp, _vp, _u64, C.c_uint32, _vp, _vp, _vp, _vp]),
            "harmonia_route_workspace_bytes": (_sz, [C.c_uint32, _u64]),
            "harmonia_route_partition": (C.c_int, [_vp, C.c_uint32, _vp, _u64, _vp, _vp, _vp, _vp, _sz, _vp]),
            "harmonia_scatter_results": (C.c_int, [_vp, _vp, _u64, _vp, _vp]),
            "harmonia_route_count": (C.c_int, [_vp, C.c_uint32, _vp, _u64, _vp, _vp, _sz, _vp]),
            "harmonia_route_push": (C.c_int, [_vp, C.c_uint32, _vp, _u64, _vp, _vp, _sz, _vp]),
            "harmonia_route_return": (C.c_int, [C.c_uint32, _vp, _u64, _vp, _vp, _sz, _vp]),
            "harmonia_segments_push": (C.c_int, [_vp, C.c_uint32, _vp, _vp, _vp, _vp, _sz, _vp]),
            "harmonia_peer_alloc": (C.c_int, [_sz, C.POINTER(_vp), _vp]),
            "harmonia_range_split_workspace_bytes": (_sz, [_u64]),
            "harmonia_range_split_count": (C.c_int, [_vp, C.c_uint32, _vp, _vp, _u64, _vp, _vp, _vp,
                                                     C.POINTER(_u64), _vp, _sz, _vp]),
            "harmonia_range_split_emit": (C.c_int, [_vp, C.c_uint32, _vp, _vp, _u64, _vp, _vp, _vp, _vp, _vp,
                                                    _sz, _vp]),
            "harmonia_range_assemble": (C.c_int, [_u64, C.c_uint32, _vp, _vp, _u64, _vp, _vp, _vp, _vp, _vp, _vp,
                                                  _vp, _vp]),
            "harmonia_peer_open": (C.c_int, [_vp, C.POINTER(_vp)]),
            "harmonia_peer_close": (C.c_int, [_vp]),
            "harmonia_peer_free": (C.c_int, [_vp]),
            "harmonia_peer_barrier": (C.c_int, [C.c_uint32, C.c_uint32, _vp, _vp, _u64, _vp, _u64, _vp]),
            "harmonia_psa_bits_auto": (C.c_int32, [_u64]),
            "harmonia_ntg_choose": (C.c_int, [_vp, _vp, C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32,
                                              C.c_uint32, C.POINTER(C.c_int32), C.POINTER(C.c_double)]),
            "harmonia_tune_group_size": (C.c_int, [_vp, _vp, C.c_uint32, C.POINTER(QueryOpts),
                                                   C.POINTER(C.c_int32), C.POINTER(C.c_double)]),
            "harmonia_query_plan": (C.c_int, [_vp, _u64, C.POINTER(QueryOpts), C.POINTER(PlanInfo)]),
            "harmonia_psa_inspect": (C.c_int, [_vp, _vp, _u64, C.POINTER(QueryOpts), _vp, _sz, _vp, _vp]),
            "harmonia_profile_enable": (None, [C.c_int]),
            "harmonia_profile_read": (C.c_int, [C.POINTER(C.c_double), C.POINTER(_u64)]),
            "harmonia_status_string": (C.c_char_p, [C.c_int]),
            "harmonia_last_cuda_error": (C.c_int, []),
            "harmonia_kernel_launches": (_u64, []),
            "harmonia_abi_version": (C.c_int, []),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def ntg_choose(prof, bucket, h: int, lev0: int, gs0: int, kpl: int = 2):
    """NTG model (Eq 3/4) over host profile counters: prof uint32[n, h, 2] of
    (r, cnt) per sample and level, bucket uint32[n] or None.  Returns (GS, [S(1), ..., S(32)])."""
    prof = np.ascontiguousarray(prof, dtype=np.uint32)
    n = prof.shape[0]
    b = None if bucket is None else np.ascontiguousarray(bucket, dtype=np.uint32)
    gs, st = C.c_int32(0), (C.c_double * 6)()
    _check(lib().harmonia_ntg_choose(prof.ctypes.data, None if b is None else b.ctypes.data, n, h, lev0, gs0, kpl,
                                     C.byref(gs), st), "harmonia_ntg_choose")
    return int(gs.value), [float(x) for x in st]


def _check(status: int, what: str):
    if status != 0:
        raise HarmoniaError(status, what)


def kernel_launches() -> int:
    return int(lib().harmonia_kernel_launches())


PROF_KINDS = ["search", "range", "psa_hist", "psa_scan", "psa_scatter", "return", "build", "update"]


def profile_enable(on: bool = True):
    """Bracket every library kernel with CUDA events on its launch stream (per class)."""
    lib().harmonia_profile_enable(1 if on else 0)


def profile_read() -> dict:
    """{class: (total_ms, launches)} since the last read (synchronises the events)."""
    ms = (C.c_double * 8)()
    n = (_u64 * 8)()
    _check(lib().harmonia_profile_read(ms, n), "harmonia_profile_read")
    return {k: (float(ms[i]), int(n[i])) for i, k in enumerate(PROF_KINDS) if n[i]}


def psa_bits_auto(n_keys: int) -> int:
    return int(lib().harmonia_psa_bits_auto(n_keys))


def _torch():
    import torch

    return torch


def _stream_ptr(stream, device):
    torch = _torch()
    s = stream if stream is not None else torch.cuda.current_stream(device)
    return C.c_void_p(s.cuda_stream)


def _as_u64_dev(t, device):
    torch = _torch()
    if isinstance(t, np.ndarray):
        t = torch.from_numpy(np.ascontiguousarray(t.astype(np.uint64, copy=False)))
    if t.dtype not in (torch.uint64, torch.int64):
        raise TypeError(f"expected uint64/int64 tensor, got {t.dtype}")
    if t.device.type != "cuda":
        t = t.to(device)
    return t.contiguous()


def make_opts(group_size=0, psa_bits=0, smem_levels=0, window=0, flags=0, lane_queries=0,
              sort_chunk=0, l2_window_bytes=0) -> QueryOpts:
    o = QueryOpts()
    o.group_size, o.psa_bits, o.smem_levels, o.flags, o.window = group_size, psa_bits, smem_levels, flags, window
    o.lane_queries = lane_queries
    o.sort_chunk = sort_chunk
    o.l2_window_bytes = l2_window_bytes
    return o


class Tree:
    """One Harmonia layout on one GPU (``harmonia_build``).

    keys / values: strictly increasing uint64 keys and their uint64 values, as CUDA tensors
    (built in place on that device) or host arrays/tensors (copied).  ``fanout`` is F,
    ``fill`` the bulk-load occupancy (C-A6)."""

    def __init__(self, keys, values, fanout: int = 64, fill: float = 1.0, device=None, stream=None):
        torch = _torch()
        self.device = torch.device(device) if device is not None else torch.device("cuda", torch.cuda.current_device())
        self._h = C.c_void_p()
        opts = BuildOpts(fanout, fill, 0, 0)
        with torch.cuda.device(self.device):
            if isinstance(keys, np.ndarray) or (hasattr(keys, "device") and keys.device.type == "cpu"):
                k = np.ascontiguousarray(np.asarray(keys if isinstance(keys, np.ndarray) else keys.numpy()).astype(np.uint64))
                v = np.ascontiguousarray(np.asarray(values if isinstance(values, np.ndarray) else values.numpy()).astype(np.uint64))
                if k.shape != v.shape:
                    raise ValueError("keys and values differ in length")
                st = _stream_ptr(stream, self.device)
                _check(lib().harmonia_build(k.ctypes.data, v.ctypes.data, k.shape[0], C.byref(opts), st,
                                            C.byref(self._h)), "harmonia_build")
            else:
                k, v = _as_u64_dev(keys, self.device), _as_u64_dev(values, self.device)
                if k.shape != v.shape:
                    raise ValueError("keys and values differ in length")
                opts.keys_on_device = 1
                st = _stream_ptr(stream, self.device)
                _check(lib().harmonia_build(k.data_ptr(), v.data_ptr(), k.numel(), C.byref(opts), st,
                                            C.byref(self._h)), "harmonia_build")
        self._ws = {}

    # ------------------------------------------------------------------ lifecycle / info
    def close(self):
        if getattr(self, "_h", None) and self._h.value:
            lib().harmonia_destroy(self._h)
            self._h = C.c_void_p()

    def __del__(self):
        try:
            self.close()
        except Exception:
            pass

    def info(self) -> dict:
        inf = Info()
        _check(lib().harmonia_get_info(self._h, C.byref(inf)), "harmonia_get_info")
        d = {f: getattr(inf, f) for f, _ in Info._fields_ if f not in ("level_start", "reserved")}
        d["level_start"] = [int(inf.level_start[i]) for i in range(inf.height + 1)]
        return d

    def tune_group_size(self, samples, opts: QueryOpts | None = None, **kw):
        """NTG static profiling on a device sample of queries (~1000): the paper's
        Eq 3/4 group size and the per-size warp step counts S(1..32).  Offline, synchronous."""
        o = opts if opts is not None else make_opts(**kw)
        gs, st = C.c_int32(0), (C.c_double * 6)()
        samples = samples.contiguous()
        _check(lib().harmonia_tune_group_size(self._h, samples.data_ptr(), samples.numel(), C.byref(o), C.byref(gs), st),
               "harmonia_tune_group_size")
        return int(gs.value), [float(x) for x in st]

    def plan(self, n: int, opts: QueryOpts | None = None, **kw) -> dict:
        o = opts if opts is not None else make_opts(**kw)
        p = PlanInfo()
        _check(lib().harmonia_query_plan(self._h, n, C.byref(o), C.byref(p)), "harmonia_query_plan")
        return {f: getattr(p, f) for f, _ in PlanInfo._fields_ if f != "reserved"}

    def export_layout(self):
        """Host copies (key_region uint64[N*F], ps uint32[I+1], leaf_values uint64[L*F])."""
        i = self.info()
        kr = np.empty(i["n_nodes"] * i["fanout"], dtype=np.uint64)
        ps = np.empty(i["n_internal"] + 1, dtype=np.uint32)
        lv = np.empty(i["n_leaves"] * i["fanout"], dtype=np.uint64)
        _check(lib().harmonia_export_layout(self._h, kr.ctypes.data, ps.ctypes.data, lv.ctypes.data),
               "harmonia_export_layout")
        return i, kr, ps, lv

    def _workspace(self, nbytes: int, stream=None):
        """Workspace for calls on `stream` (the C ABI needs one per stream).  Cached per stream
        and allocated while that stream is current, so the caching allocator never hands the
        block to another stream while a kernel may still use it."""
        torch = _torch()
        if nbytes == 0:
            return None
        s = stream if stream is not None else torch.cuda.current_stream(self.device)
        key = int(s.cuda_stream)
        w = self._ws.get(key)
        if w is None or w.numel() < nbytes:
            with torch.cuda.stream(s):
                w = torch.empty(nbytes, dtype=torch.uint8, device=self.device)
            self._ws[key] = w
        return w

    # ------------------------------------------------------------------ queries
    def search(self, q, out=None, *, opts: QueryOpts | None = None, stream=None, **kw):
        """Point queries (harmonia_search_batch): value or NOT_FOUND per query."""
        torch = _torch()
        q = _as_u64_dev(q, self.device)
        n = q.numel()
        if out is None:
            out = torch.empty(n, dtype=torch.uint64, device=self.device)
        o = opts if opts is not None else make_opts(**kw)
        ws_b = lib().harmonia_search_workspace_bytes(self._h, n, C.byref(o))
        ws = self._workspace(ws_b, stream)
        st = _stream_ptr(stream, self.device)
        _check(lib().harmonia_search_batch(self._h, q.data_ptr(), n, out.data_ptr(),
                                           ws.data_ptr() if ws is not None else None, ws_b, C.byref(o), st),
               "harmonia_search_batch")
        return out

    def search_addr(self, q_addr: int, n: int, out, *, opts: QueryOpts | None = None, stream=None, **kw):
        """Point queries read from a raw device address (e.g. a peer-mapped receive buffer)."""
        o = opts if opts is not None else make_opts(**kw)
        ws_b = lib().harmonia_search_workspace_bytes(self._h, n, C.byref(o))
        ws = self._workspace(ws_b, stream)
        _check(lib().harmonia_search_batch(self._h, q_addr, n, out.data_ptr(),
                                           ws.data_ptr() if ws is not None else None, ws_b, C.byref(o),
                                           _stream_ptr(stream, self.device)), "harmonia_search_batch")
        return out

    def psa_inspect(self, q, *, opts: QueryOpts | None = None, stream=None, **kw):
        """The queries in the order the search kernel visits them after PSA (harmonia_psa_inspect)."""
        torch = _torch()
        q = _as_u64_dev(q, self.device)
        n = q.numel()
        out = torch.empty(n, dtype=torch.uint64, device=self.device)
        o = opts if opts is not None else make_opts(**kw)
        ws_b = lib().harmonia_search_workspace_bytes(self._h, n, C.byref(o))
        ws = self._workspace(ws_b, stream)
        _check(lib().harmonia_psa_inspect(self._h, q.data_ptr(), n, C.byref(o),
                                          ws.data_ptr() if ws is not None else None, ws_b, out.data_ptr(),
                                          _stream_ptr(stream, self.device)), "harmonia_psa_inspect")
        return out

    def search_host(self, q_host, out_host=None, *, opts: QueryOpts | None = None, stream=None, **kw):
        """End-to-end point queries from host memory (pinned CPU tensors for overlap).
        Asynchronous on `stream`, like harmonia_search_batch_host: synchronise the stream
        before reading the returned host buffer."""
        torch = _torch()
        if isinstance(q_host, np.ndarray):
            q_host = torch.from_numpy(np.ascontiguousarray(q_host.astype(np.uint64, copy=False)))
        assert q_host.device.type == "cpu"
        n = q_host.numel()
        if out_host is None:
            out_host = torch.empty(n, dtype=torch.uint64, pin_memory=True)
        o = opts if opts is not None else make_opts(**kw)
        ws_b = lib().harmonia_search_host_workspace_bytes(self._h, n, C.byref(o))
        ws = self._workspace(ws_b, stream)
        st = _stream_ptr(stream, self.device)
        _check(lib().harmonia_search_batch_host(self._h, q_host.data_ptr(), n, out_host.data_ptr(),
                                                ws.data_ptr(), ws_b, C.byref(o), st), "harmonia_search_batch_host")
        return out_host

    def range(self, lo, hi, cap: int, *, out=None, opts: QueryOpts | None = None, stream=None, **kw):
        """Inclusive range queries: (keys [n, cap], values [n, cap], counts [n] uint32).
        Without `out`, fresh slabs pre-filled with PAD / NOT_FOUND are returned; with
        out=(keys, values, counts) those buffers are written as the C ABI does (slab entries
        past a range's count are left untouched)."""
        torch = _torch()
        lo, hi = _as_u64_dev(lo, self.device), _as_u64_dev(hi, self.device)
        n = lo.numel()
        if out is not None:
            ko, vo, cnt = out
        else:
            ko = torch.full((n, cap), KEY_PAD, dtype=torch.uint64, device=self.device) if cap else None
            vo = torch.full((n, cap), NOT_FOUND, dtype=torch.uint64, device=self.device) if cap else None
            cnt = torch.empty(n, dtype=torch.uint32, device=self.device)
        o = opts if opts is not None else make_opts(**kw)
        ws_b = lib().harmonia_range_workspace_bytes(self._h, n, C.byref(o))
        ws = self._workspace(ws_b, stream)
        st = _stream_ptr(stream, self.device)
        _check(lib().harmonia_range_batch(self._h, lo.data_ptr(), hi.data_ptr(), n, cap,
                                          ko.data_ptr() if ko is not None else None,
                                          vo.data_ptr() if vo is not None else None, cnt.data_ptr(),
                                          ws.data_ptr() if ws is not None else None, ws_b, C.byref(o), st),
               "harmonia_range_batch")
        return ko, vo, cnt

    def last_update_mode(self) -> int:
        """1 if the last update batch ran in place, 2 if it rebuilt the layout (0: none yet)."""
        return int(lib().harmonia_update_last_mode(self._h))

    def update(self, ops, keys, values, seq=None, stream=None):
        """Batched upsert (op 0) / delete (op 1), sequential semantics in batch order (or in
        ascending `seq`, uint64 per op, when given: harmonia_update_batch_seq)."""
        torch = _torch()
        if isinstance(ops, np.ndarray):
            ops = torch.from_numpy(np.ascontiguousarray(ops.astype(np.uint8)))
        ops = ops.to(self.device, dtype=torch.uint8).contiguous()
        keys, values = _as_u64_dev(keys, self.device), _as_u64_dev(values, self.device)
        n = keys.numel()
        ws_b = lib().harmonia_update_workspace_bytes(self._h, n)
        ws = torch.empty(max(ws_b, 1), dtype=torch.uint8, device=self.device)
        st = _stream_ptr(stream, self.device)
        if seq is None:
            _check(lib().harmonia_update_batch(self._h, ops.data_ptr(), keys.data_ptr(), values.data_ptr(), n,
                                               ws.data_ptr(), ws_b, st), "harmonia_update_batch")
        else:
            seq = _as_u64_dev(seq, self.device)
            _check(lib().harmonia_update_batch_seq(self._h, ops.data_ptr(), keys.data_ptr(), values.data_ptr(),
                                                   seq.data_ptr(), n, ws.data_ptr(), ws_b, st),
                   "harmonia_update_batch_seq")


def update_validate(ops, keys, values, stream=None):
    """harmonia_update_validate: a device uint32[1] holding 0 for a valid update batch, else
    2 (reserved key/value) | 4 (bad op code)."""
    torch = _torch()
    dev = keys.device
    flags = torch.empty(1, dtype=torch.int32, device=dev)
    _check(lib().harmonia_update_validate(ops.data_ptr(), keys.data_ptr(), values.data_ptr(), keys.numel(),
                                          flags.data_ptr(), _stream_ptr(stream, dev)), "harmonia_update_validate")
    return flags


def route_partition(splitters, P: int, q, stream=None):
    """Group queries by destination shard: returns (routed, pos, counts list)."""
    torch = _torch()
    dev = q.device
    n = q.numel()
    routed = torch.empty(n, dtype=torch.uint64, device=dev)
    pos = torch.empty(n, dtype=torch.uint32, device=dev)
    counts = (C.c_uint64 * P)()
    ws_b = lib().harmonia_route_workspace_bytes(P, n)
    ws = torch.empty(max(ws_b, 1), dtype=torch.uint8, device=dev)
    sp = splitters.data_ptr() if P > 1 else None
    _check(lib().harmonia_route_partition(sp, P, q.data_ptr(), n, routed.data_ptr(), pos.data_ptr(), counts,
                                          ws.data_ptr(), ws_b, _stream_ptr(stream, dev)), "harmonia_route_partition")
    return routed, pos, [int(c) for c in counts]


def route_update_payload(ops, values, pos, rank: int, stream=None):
    """Routed update payload (harmonia_route_update_payload): ops/values in routed order and the
    global sequence number rank << 32 | original position of every routed op."""
    torch = _torch()
    n = pos.numel()
    o = torch.empty(n, dtype=torch.uint8, device=pos.device)
    v = torch.empty(n, dtype=torch.uint64, device=pos.device)
    sq = torch.empty(n, dtype=torch.uint64, device=pos.device)
    _check(lib().harmonia_route_update_payload(ops.data_ptr(), values.data_ptr(), pos.data_ptr(), n, rank,
                                               o.data_ptr(), v.data_ptr(), sq.data_ptr(),
                                               _stream_ptr(stream, pos.device)), "harmonia_route_update_payload")
    return o, v, sq


def scatter_results(vals, pos, out=None, stream=None):
    torch = _torch()
    n = vals.numel()
    if out is None:
        out = torch.empty(n, dtype=torch.uint64, device=vals.device)
    _check(lib().harmonia_scatter_results(vals.data_ptr(), pos.data_ptr(), n, out.data_ptr(),
                                          _stream_ptr(stream, vals.device)), "harmonia_scatter_results")
    return out


# ----------------------------------------------------------------------------- fused routing
def _u64_array(vals):
    a = (C.c_uint64 * max(len(vals), 1))()
    for i, v in enumerate(vals):
        a[i] = int(v) & ((1 << 64) - 1)
    return a


def route_workspace(P: int, n: int, device):
    """Workspace for one batch of the fused-routing calls (kept for the whole batch)."""
    torch = _torch()
    b = lib().harmonia_route_workspace_bytes(P, n)
    return torch.empty(b, dtype=torch.uint8, device=device)


def route_count(splitters, P: int, q, ws, stream=None) -> list:
    """Destination counts of the batch (harmonia_route_count; ranks kept in ws)."""
    counts = (C.c_uint64 * P)()
    sp = splitters.data_ptr() if P > 1 else None
    _check(lib().harmonia_route_count(sp, P, q.data_ptr(), q.numel(), counts, ws.data_ptr(), ws.numel(),
                                      _stream_ptr(stream, q.device)), "harmonia_route_count")
    return [int(c) for c in counts]


def route_push(splitters, P: int, q, dst_addrs, ws, stream=None):
    """Write destination d's run of the batch to device address dst_addrs[d] (harmonia_route_push)."""
    sp = splitters.data_ptr() if P > 1 else None
    _check(lib().harmonia_route_push(sp, P, q.data_ptr(), q.numel(), _u64_array(dst_addrs), ws.data_ptr(),
                                     ws.numel(), _stream_ptr(stream, q.device)), "harmonia_route_push")


def route_return(P: int, back_addr: int, n: int, out, ws, stream=None):
    """out[i] = back[routed position of query i] (harmonia_route_return)."""
    _check(lib().harmonia_route_return(P, back_addr, n, out.data_ptr(), ws.data_ptr(), ws.numel(),
                                       _stream_ptr(stream, out.device)), "harmonia_route_return")
    return out


def segments_push(src, src_off, lens, dst_addrs, ws, stream=None):
    """Copy src[src_off[s] : +lens[s]] to device address dst_addrs[s] for every segment."""
    _check(lib().harmonia_segments_push(src.data_ptr(), len(lens), _u64_array(src_off), _u64_array(lens),
                                        _u64_array(dst_addrs), ws.data_ptr(), ws.numel(),
                                        _stream_ptr(stream, src.device)), "harmonia_segments_push")


class PeerBuffer:
    """A device buffer other processes can map (CUDA IPC, harmonia_peer_alloc/open)."""

    def __init__(self, nbytes: int):
        self.ptr, self.nbytes = C.c_void_p(), nbytes
        self.handle = (C.c_char * 64)()
        _check(lib().harmonia_peer_alloc(nbytes, C.byref(self.ptr), self.handle), "harmonia_peer_alloc")

    @property
    def addr(self) -> int:
        return int(self.ptr.value)

    def handle_bytes(self) -> bytes:
        return bytes(self.handle)

    @staticmethod
    def open(handle: bytes) -> int:
        p = C.c_void_p()
        h = (C.c_char * 64).from_buffer_copy(handle)
        _check(lib().harmonia_peer_open(h, C.byref(p)), "harmonia_peer_open")
        return int(p.value)

    @staticmethod
    def close_mapping(addr: int):
        _check(lib().harmonia_peer_close(C.c_void_p(addr)), "harmonia_peer_close")

    def free(self):
        if self.ptr.value:
            _check(lib().harmonia_peer_free(self.ptr), "harmonia_peer_free")
            self.ptr = C.c_void_p()


def peer_barrier(P: int, me: int, flag_addrs, my_flags_addr: int, epoch: int, error, timeout_ns: int = 0,
                 stream=None):
    """harmonia_peer_barrier: device-side barrier of the fused routing (asynchronous; `flag_addrs`
    a device uint64 tensor of the P ranks' flag-array addresses, `error` a device int32[1])."""
    _check(lib().harmonia_peer_barrier(P, me, flag_addrs.data_ptr(), my_flags_addr, epoch, error.data_ptr(),
                                       timeout_ns, _stream_ptr(stream, error.device)), "harmonia_peer_barrier")


# ----------------------------------------------------------------------------- range routing
def range_split(splitters, P: int, lo, hi, stream=None):
    """Cut ranges at the shard splitters (harmonia_range_split_count + _emit).
    Returns (plo, phi, pid, counts per destination, pbase): the pieces destination-major."""
    torch = _torch()
    dev, n = lo.device, lo.numel()
    npieces = torch.empty(n + 1, dtype=torch.uint32, device=dev)
    pbase = torch.empty(n + 1, dtype=torch.uint32, device=dev)
    ws_b = lib().harmonia_range_split_workspace_bytes(n)
    ws = torch.empty(ws_b, dtype=torch.uint8, device=dev)
    counts, total = (C.c_uint64 * P)(), C.c_uint64(0)
    sp = splitters.data_ptr() if P > 1 else None
    st = _stream_ptr(stream, dev)
    _check(lib().harmonia_range_split_count(sp, P, lo.data_ptr(), hi.data_ptr(), n, npieces.data_ptr(),
                                            pbase.data_ptr(), counts, C.byref(total), ws.data_ptr(), ws_b, st),
           "harmonia_range_split_count")
    m = int(total.value)
    plo = torch.empty(m, dtype=torch.uint64, device=dev)
    phi = torch.empty(m, dtype=torch.uint64, device=dev)
    pid = torch.empty(m, dtype=torch.uint32, device=dev)
    if n:
        _check(lib().harmonia_range_split_emit(sp, P, lo.data_ptr(), hi.data_ptr(), n, pbase.data_ptr(),
                                               plo.data_ptr(), phi.data_ptr(), pid.data_ptr(), ws.data_ptr(), ws_b,
                                               st), "harmonia_range_split_emit")
    return plo, phi, pid, [int(c) for c in counts], pbase


def range_assemble(n: int, cap: int, pbase, pid, counts, keys, values, stream=None):
    """Reassemble routed range answers (harmonia_range_assemble): (keys [n, cap], values [n, cap],
    totals [n] uint64); slab entries past a range's count hold PAD / NOT_FOUND."""
    torch = _torch()
    dev = pbase.device
    m = pid.numel()
    ko = torch.full((n, cap), KEY_PAD, dtype=torch.uint64, device=dev) if cap else None
    vo = torch.full((n, cap), NOT_FOUND, dtype=torch.uint64, device=dev) if cap else None
    tot = torch.empty(n, dtype=torch.uint64, device=dev)
    rows = torch.empty(max(m, 1), dtype=torch.uint32, device=dev)
    _check(lib().harmonia_range_assemble(n, cap, pbase.data_ptr(), pid.data_ptr() if m else None, m,
                                         counts.data_ptr() if m else None,
                                         keys.data_ptr() if (cap and m) else None,
                                         values.data_ptr() if (cap and m) else None, rows.data_ptr(),
                                         ko.data_ptr() if cap else None, vo.data_ptr() if cap else None,
                                         tot.data_ptr(), _stream_ptr(stream, dev)), "harmonia_range_assemble")
    return ko, vo, tot
