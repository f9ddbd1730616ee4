"""CPU oracle for Harmonia (PPoPP'19) — ctypes front end of ``oracle/liboracle.so``.

TEST INFRASTRUCTURE ONLY.  Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` legs may import this package.  The product package
(``paper_conf_ppopp_yanlpz19_b200``) never imports it, and this package never imports the
product: they share no code.

Every function here is a thin marshalling wrapper over the C++ functions declared in
``oracle/oracle.h``; the citations and parity-pin notes live there.
"""
from __future__ import annotations

import ctypes as C
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")
SOURCES = ["sorted_array.cc", "bptree.cc", "layout.cc", "model.cc"]

NOT_FOUND = np.uint64(0xFFFFFFFFFFFFFFFF)
PAD = np.uint64(0xFFFFFFFFFFFFFFFF)


def build(force: bool = False) -> str:
    """Compile liboracle.so with g++ (no CUDA involved)."""
    srcs = [os.path.join(_HERE, s) for s in SOURCES]
    hdr = os.path.join(_HERE, "oracle.h")
    if not force and os.path.exists(LIB_PATH):
        mt = os.path.getmtime(LIB_PATH)
        if all(os.path.getmtime(s) <= mt for s in srcs + [hdr]):
            return LIB_PATH
    tmp = LIB_PATH + f".tmp{os.getpid()}"
    cmd = ["g++", "-O2", "-std=c++17", "-shared", "-fPIC", "-pthread", "-o", tmp] + srcs
    subprocess.check_call(cmd)
    os.replace(tmp, LIB_PATH)
    return LIB_PATH


_lib = None

u64p = C.POINTER(C.c_uint64)
u32p = C.POINTER(C.c_uint32)
u8p = C.POINTER(C.c_uint8)


def lib():
    global _lib
    if _lib is None:
        build()
        L = C.CDLL(LIB_PATH)
        sig = {
            "orc_sorted_search": (None, [u64p, u64p, C.c_uint64, u64p, C.c_uint64, u64p, C.c_int]),
            "orc_sorted_range": (None, [u64p, u64p, C.c_uint64, u64p, u64p, C.c_uint64, C.c_uint32,
                                        u64p, u64p, u32p, C.c_int]),
            "orc_brute_search": (None, [u64p, u64p, C.c_uint64, u64p, C.c_uint64, u64p]),
            "orc_brute_range": (None, [u64p, u64p, C.c_uint64, u64p, u64p, C.c_uint64, C.c_uint32,
                                       u64p, u64p, u32p]),
            "orc_bpt_create": (C.c_void_p, [C.c_uint32]),
            "orc_bpt_destroy": (None, [C.c_void_p]),
            "orc_bpt_insert": (C.c_int, [C.c_void_p, C.c_uint64, C.c_uint64]),
            "orc_bpt_erase": (C.c_int, [C.c_void_p, C.c_uint64]),
            "orc_bpt_search": (None, [C.c_void_p, u64p, C.c_uint64, u64p]),
            "orc_bpt_search_mt": (None, [C.c_void_p, u64p, C.c_uint64, u64p, C.c_int]),
            "orc_bpt_insert_array": (C.c_uint64, [C.c_void_p, u64p, u64p, C.c_uint64]),
            "orc_bpt_range": (None, [C.c_void_p, u64p, u64p, C.c_uint64, C.c_uint32, u64p, u64p, u32p]),
            "orc_bpt_size": (C.c_uint64, [C.c_void_p]),
            "orc_bpt_height": (C.c_uint32, [C.c_void_p]),
            "orc_bpt_check": (C.c_int, [C.c_void_p]),
            "orc_bpt_debug_mutate": (C.c_int, [C.c_void_p, C.c_int]),
            "orc_bpt_dump": (None, [C.c_void_p, u64p, u64p]),
            "orc_bpt_level_stats": (None, [C.c_void_p, u64p, u64p, C.c_uint32]),
            "orc_bpt_quarter_stats": (None, [C.c_void_p, u64p, C.c_uint64, u64p]),
            "orc_bpt_comparisons": (None, [C.c_void_p, u64p, C.c_uint64, u32p]),
            "orc_layout_shape": (C.c_uint32, [C.c_uint64, C.c_uint32, C.c_double, u64p]),
            "orc_layout_build": (C.c_int, [u64p, u64p, C.c_uint64, C.c_uint32, C.c_double, u64p, u32p, u64p]),
            "orc_layout_check": (C.c_int, [u64p, u32p, u64p, C.c_uint32, C.c_uint32, u64p, u64p, u64p,
                                           C.c_uint64, C.c_char_p, C.c_int]),
            "orc_layout_check2": (C.c_int, [u64p, u32p, u64p, C.c_uint32, C.c_uint32, u64p, u64p, u64p,
                                            C.c_uint64, C.c_char_p, C.c_int, C.c_int]),
            "orc_layout_search": (None, [u64p, u32p, u64p, C.c_uint32, C.c_uint32, u64p, u64p, C.c_uint64, u64p]),
            "orc_layout_range": (None, [u64p, u32p, u64p, C.c_uint32, C.c_uint32, u64p, u64p, u64p, C.c_uint64,
                                        C.c_uint32, u64p, u64p, u32p]),
            "orc_eq1_child": (C.c_uint64, [u32p, C.c_uint64, C.c_uint64]),
            "orc_psa_bits": (C.c_uint32, [C.c_uint32, C.c_double, C.c_uint32]),
            "orc_psa_bucket": (C.c_uint64, [C.c_uint64, C.c_uint32, C.c_uint64, C.c_uint64]),
            "orc_psa_buckets": (None, [u64p, C.c_uint64, C.c_uint32, C.c_uint64, C.c_uint64, u64p]),
            "orc_psa_order": (None, [u64p, C.c_uint64, C.c_uint32, C.c_uint64, C.c_uint64, u64p]),
            "orc_ntg_steps": (C.c_uint32, [C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32]),
            "orc_ntg_warp_steps": (C.c_double, [u64p, u32p, C.c_uint32, C.c_uint32, u64p, u64p, C.c_uint64,
                                                C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32]),
            "orc_ntg_choose_gs": (C.c_uint32, [u64p, u32p, C.c_uint32, C.c_uint32, u64p, u64p, C.c_uint64,
                                               C.c_uint32, C.c_uint32, C.c_uint32, C.c_uint32]),
            "orc_warp_transactions": (C.c_double, [u64p, u32p, C.c_uint32, C.c_uint32, u64p, u64p,
                                                   C.c_uint64, C.c_uint32]),
            "orc_map_create": (C.c_void_p, [u64p, u64p, C.c_uint64]),
            "orc_map_destroy": (None, [C.c_void_p]),
            "orc_map_apply": (C.c_uint64, [C.c_void_p, u8p, u64p, u64p, C.c_uint64]),
            "orc_map_dump": (C.c_uint64, [C.c_void_p, u64p, u64p, C.c_uint64]),
        }
        for name, (res, args) in sig.items():
            f = getattr(L, name)
            f.restype = res
            f.argtypes = args
        _lib = L
    return _lib


def _p64(a: np.ndarray):
    assert a.dtype == np.uint64 and a.flags.c_contiguous, (a.dtype, a.flags)
    return a.ctypes.data_as(u64p)


def _p32(a: np.ndarray):
    assert a.dtype == np.uint32 and a.flags.c_contiguous
    return a.ctypes.data_as(u32p)


def _u64(a) -> np.ndarray:
    return np.ascontiguousarray(np.asarray(a, dtype=np.uint64))


# ----------------------------------------------------------------------------- O1 / O3
def sorted_search(keys, vals, q, nthreads: int = 0) -> np.ndarray:
    keys, vals, q = _u64(keys), _u64(vals), _u64(q)
    out = np.empty(q.shape[0], dtype=np.uint64)
    lib().orc_sorted_search(_p64(keys), _p64(vals), keys.shape[0], _p64(q), q.shape[0], _p64(out), nthreads)
    return out


def _range_out(nq, cap):
    return (np.zeros(nq * cap, dtype=np.uint64), np.zeros(nq * cap, dtype=np.uint64),
            np.zeros(nq, dtype=np.uint32))


def sorted_range(keys, vals, lo, hi, cap: int, nthreads: int = 0):
    keys, vals, lo, hi = _u64(keys), _u64(vals), _u64(lo), _u64(hi)
    ko, vo, cnt = _range_out(lo.shape[0], cap)
    lib().orc_sorted_range(_p64(keys), _p64(vals), keys.shape[0], _p64(lo), _p64(hi), lo.shape[0], cap,
                           _p64(ko), _p64(vo), _p32(cnt), nthreads)
    return ko.reshape(-1, cap) if cap else ko, vo.reshape(-1, cap) if cap else vo, cnt


def brute_search(keys, vals, q) -> np.ndarray:
    keys, vals, q = _u64(keys), _u64(vals), _u64(q)
    out = np.empty(q.shape[0], dtype=np.uint64)
    lib().orc_brute_search(_p64(keys), _p64(vals), keys.shape[0], _p64(q), q.shape[0], _p64(out))
    return out


def brute_range(keys, vals, lo, hi, cap: int):
    keys, vals, lo, hi = _u64(keys), _u64(vals), _u64(lo), _u64(hi)
    ko, vo, cnt = _range_out(lo.shape[0], cap)
    lib().orc_brute_range(_p64(keys), _p64(vals), keys.shape[0], _p64(lo), _p64(hi), lo.shape[0], cap,
                          _p64(ko), _p64(vo), _p32(cnt))
    return ko.reshape(-1, cap) if cap else ko, vo.reshape(-1, cap) if cap else vo, cnt


# ----------------------------------------------------------------------------- O2
class BPlusTree:
    """The paper's regular pointer B+tree."""

    def __init__(self, fanout: int):
        self.F = fanout
        self._h = lib().orc_bpt_create(fanout)

    def __del__(self):
        if getattr(self, "_h", None):
            lib().orc_bpt_destroy(self._h)
            self._h = None

    def insert(self, k, v) -> int:
        return lib().orc_bpt_insert(self._h, int(k), int(v))

    def insert_many(self, keys, vals):
        k, v = _u64(keys), _u64(vals)
        return int(lib().orc_bpt_insert_array(self._h, _p64(k), _p64(v), k.shape[0]))

    def erase(self, k) -> int:
        return lib().orc_bpt_erase(self._h, int(k))

    def search(self, q, nthreads: int = 1) -> np.ndarray:
        q = _u64(q)
        out = np.empty(q.shape[0], dtype=np.uint64)
        if nthreads == 1:
            lib().orc_bpt_search(self._h, _p64(q), q.shape[0], _p64(out))
        else:
            lib().orc_bpt_search_mt(self._h, _p64(q), q.shape[0], _p64(out), nthreads)
        return out

    def range(self, lo, hi, cap: int):
        lo, hi = _u64(lo), _u64(hi)
        ko, vo, cnt = _range_out(lo.shape[0], cap)
        lib().orc_bpt_range(self._h, _p64(lo), _p64(hi), lo.shape[0], cap, _p64(ko), _p64(vo), _p32(cnt))
        return ko.reshape(-1, cap) if cap else ko, vo.reshape(-1, cap) if cap else vo, cnt

    def __len__(self):
        return int(lib().orc_bpt_size(self._h))

    @property
    def height(self) -> int:
        return int(lib().orc_bpt_height(self._h))

    def check(self) -> int:
        return int(lib().orc_bpt_check(self._h))

    def debug_mutate(self, kind: int) -> bool:
        """Test hook: corrupt the tree one way (bptree.cc orc_bpt_debug_mutate)."""
        return bool(lib().orc_bpt_debug_mutate(self._h, kind))

    def dump(self):
        n = len(self)
        k = np.empty(n, dtype=np.uint64)
        v = np.empty(n, dtype=np.uint64)
        lib().orc_bpt_dump(self._h, _p64(k), _p64(v))
        return k, v

    def level_stats(self, maxlev: int = 64):
        nodes = np.zeros(maxlev, dtype=np.uint64)
        ent = np.zeros(maxlev, dtype=np.uint64)
        lib().orc_bpt_level_stats(self._h, _p64(nodes), _p64(ent), maxlev)
        h = self.height
        return nodes[:h], ent[:h]

    def quarter_stats(self, q) -> np.ndarray:
        q = _u64(q)
        c = np.zeros(4, dtype=np.uint64)
        lib().orc_bpt_quarter_stats(self._h, _p64(q), q.shape[0], _p64(c))
        return c

    def comparisons(self, q) -> np.ndarray:
        q = _u64(q)
        h = self.height
        out = np.zeros(q.shape[0] * h, dtype=np.uint32)
        lib().orc_bpt_comparisons(self._h, _p64(q), q.shape[0], _p32(out))
        return out.reshape(-1, h)


# ----------------------------------------------------------------------------- O4
class Layout:
    """A Harmonia layout held on the host (oracle-built or exported from the GPU)."""

    def __init__(self, fanout, height, level_start, key_region, ps, leaf_vals):
        self.F = int(fanout)
        self.h = int(height)
        self.level_start = _u64(level_start)
        self.key_region = _u64(key_region)
        self.ps = np.ascontiguousarray(np.asarray(ps, dtype=np.uint32))
        self.leaf_vals = _u64(leaf_vals)

    @property
    def n_nodes(self):
        return int(self.level_start[self.h])

    @property
    def n_internal(self):
        return int(self.level_start[self.h - 1])

    def check(self, keys, vals, strict_separators: bool = True):
        """I1-I7 against the record set; strict_separators=False drops the equality half of I5
        (separator == subtree minimum), which only a fresh build guarantees."""
        keys, vals = _u64(keys), _u64(vals)
        msg = C.create_string_buffer(256)
        r = lib().orc_layout_check2(_p64(self.key_region), _p32(self.ps), _p64(self.leaf_vals), self.F, self.h,
                                    _p64(self.level_start), _p64(keys), _p64(vals), keys.shape[0], msg, 256,
                                    1 if strict_separators else 0)
        return int(r), msg.value.decode()

    def search(self, q) -> np.ndarray:
        q = _u64(q)
        out = np.empty(q.shape[0], dtype=np.uint64)
        lib().orc_layout_search(_p64(self.key_region), _p32(self.ps), _p64(self.leaf_vals), self.F, self.h,
                                _p64(self.level_start), _p64(q), q.shape[0], _p64(out))
        return out

    def range(self, lo, hi, cap: int):
        lo, hi = _u64(lo), _u64(hi)
        ko, vo, cnt = _range_out(lo.shape[0], cap)
        lib().orc_layout_range(_p64(self.key_region), _p32(self.ps), _p64(self.leaf_vals), self.F, self.h,
                               _p64(self.level_start), _p64(lo), _p64(hi), lo.shape[0], cap,
                               _p64(ko), _p64(vo), _p32(cnt))
        return ko.reshape(-1, cap) if cap else ko, vo.reshape(-1, cap) if cap else vo, cnt

    def _args(self):
        return (_p64(self.key_region), _p32(self.ps), self.F, self.h, _p64(self.level_start))

    def ntg_warp_steps(self, q, gs, kpl=2, lev0=0, warp=32) -> float:
        q = _u64(q)
        kr, ps, F, h, ls = self._args()
        return float(lib().orc_ntg_warp_steps(kr, ps, F, h, ls, _p64(q), q.shape[0], gs, kpl, lev0, warp))

    def ntg_choose_gs(self, q, gs0, kpl=2, lev0=0, warp=32) -> int:
        q = _u64(q)
        kr, ps, F, h, ls = self._args()
        return int(lib().orc_ntg_choose_gs(kr, ps, F, h, ls, _p64(q), q.shape[0], gs0, kpl, lev0, warp))

    def warp_transactions(self, q, queries_per_warp) -> float:
        q = _u64(q)
        kr, ps, F, h, ls = self._args()
        return float(lib().orc_warp_transactions(kr, ps, F, h, ls, _p64(q), q.shape[0], queries_per_warp))


def layout_shape(n: int, fanout: int, fill: float = 1.0):
    ln = np.zeros(64, dtype=np.uint64)
    h = lib().orc_layout_shape(n, fanout, fill, _p64(ln))
    return int(h), ln[:h].copy()


def layout_build(keys, vals, fanout: int, fill: float = 1.0) -> Layout:
    keys, vals = _u64(keys), _u64(vals)
    h, ln = layout_shape(keys.shape[0], fanout, fill)
    ls = np.zeros(h + 1, dtype=np.uint64)
    ls[1:] = np.cumsum(ln)
    N, I, L = int(ls[h]), int(ls[h - 1]), int(ln[h - 1])
    kr = np.empty(N * fanout, dtype=np.uint64)
    ps = np.empty(I + 1, dtype=np.uint32)
    lv = np.empty(L * fanout, dtype=np.uint64)
    r = lib().orc_layout_build(_p64(keys), _p64(vals), keys.shape[0], fanout, fill, _p64(kr), _p32(ps), _p64(lv))
    assert r == 0
    return Layout(fanout, h, ls, kr, ps, lv)


def eq1_child(ps, node_idx: int, i: int) -> int:
    ps = np.ascontiguousarray(np.asarray(ps, dtype=np.uint32))
    return int(lib().orc_eq1_child(_p32(ps), node_idx, i))


# ----------------------------------------------------------------------------- O5
def psa_bits(B: int, T: float, K: int) -> int:
    return int(lib().orc_psa_bits(B, float(T), K))


def psa_bucket(q: int, nbits: int, min_key: int, max_key: int) -> int:
    return int(lib().orc_psa_bucket(int(q), nbits, int(min_key), int(max_key)))


def psa_buckets(q, nbits: int, min_key: int, max_key: int) -> np.ndarray:
    """orc_psa_bucket of every query (C-A11)."""
    q = _u64(q)
    out = np.empty(q.shape[0], dtype=np.uint64)
    lib().orc_psa_buckets(_p64(q), q.shape[0], nbits, min_key, max_key, _p64(out))
    return out


def psa_order(q, nbits: int, min_key: int, max_key: int) -> np.ndarray:
    q = _u64(q)
    perm = np.empty(q.shape[0], dtype=np.uint64)
    lib().orc_psa_order(_p64(q), q.shape[0], nbits, int(min_key), int(max_key), _p64(perm))
    return perm


def ntg_steps(r: int, cnt: int, gs: int, kpl: int = 1) -> int:
    return int(lib().orc_ntg_steps(r, cnt, gs, kpl))


# ----------------------------------------------------------------------------- O6
class UpdateMap:
    def __init__(self, keys, vals):
        keys, vals = _u64(keys), _u64(vals)
        self._h = lib().orc_map_create(_p64(keys), _p64(vals), keys.shape[0])

    def __del__(self):
        if getattr(self, "_h", None):
            lib().orc_map_destroy(self._h)
            self._h = None

    def apply(self, ops, keys, vals) -> int:
        ops = np.ascontiguousarray(np.asarray(ops, dtype=np.uint8))
        keys, vals = _u64(keys), _u64(vals)
        return int(lib().orc_map_apply(self._h, ops.ctypes.data_as(u8p), _p64(keys), _p64(vals), keys.shape[0]))

    def dump(self):
        n = int(lib().orc_map_dump(self._h, None, None, 0))
        k = np.empty(n, dtype=np.uint64)
        v = np.empty(n, dtype=np.uint64)
        lib().orc_map_dump(self._h, _p64(k), _p64(v), n)
        return k, v
