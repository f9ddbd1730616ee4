"""Seeded, counter-based input generators shared by the tests, the oracle and the bench.

This module holds NONE of the method's arithmetic (no layout, no search, no PSA): it only
draws key sets, values, query batches, range batches and update batches, with the shapes
and distributions of the paper's workloads (uniform queries over trees of
2^23..2^26 64-bit keys; batches of 4096K updates, 5 % inserts + 95 % updates) plus the
north_star's Zipfian and sorted-run sets.  The recipe is stated in DESIGN.md §5.

Everything is a pure function of (seed, index) via splitmix64, so any slice of any
stream can be regenerated independently (shardable across ranks).
"""
from __future__ import annotations

import functools

import numpy as np

SEED = 0x4841524D4F4E4941  # "HARMONIA"
SEED_KEY, SEED_VAL, SEED_QUERY, SEED_RANGE, SEED_OPS = (SEED + i for i in range(5))
U64_MAX = np.uint64(0xFFFFFFFFFFFFFFFF)
_M64 = (1 << 64) - 1


def splitmix64(x) -> np.ndarray:
    """splitmix64 finaliser over a uint64 array (wrapping arithmetic)."""
    x = np.asarray(x, dtype=np.uint64)
    with np.errstate(over="ignore"):
        x = x + np.uint64(0x9E3779B97F4A7C15)
        z = (x ^ (x >> np.uint64(30))) * np.uint64(0xBF58476D1CE4E5B9)
        z = (z ^ (z >> np.uint64(27))) * np.uint64(0x94D049BB133111EB)
        return z ^ (z >> np.uint64(31))


def _stream(seed: int, start: int, n: int) -> np.ndarray:
    idx = np.arange(start, start + n, dtype=np.uint64)
    return splitmix64(np.uint64(seed & _M64) ^ idx)


def _unit(seed: int, start: int, n: int) -> np.ndarray:
    """Uniform doubles in [0, 1) from the top 53 bits of the stream."""
    return (_stream(seed, start, n) >> np.uint64(11)).astype(np.float64) * (1.0 / (1 << 53))


# ------------------------------------------------------------------------------ keys
def uniform_keys(T: int, seed: int = SEED_KEY, start: int = 0, count: int | None = None) -> np.ndarray:
    """Jittered-stride keys: key_i = i*D + (h(i) mod D), D = floor((2^64-2)/T).

    Strictly increasing, unique, never UINT64_MAX, stratified-uniform over 64 bits (so the
    most significant bits are uniform, as Eq 2's analysis assumes).  ``start`` /
    ``count`` generate the slice [start, start+count) of the same set.
    """
    if count is None:
        count = T - start
    if T == 0 or count == 0:
        return np.zeros(0, dtype=np.uint64)
    D = np.uint64(((1 << 64) - 2) // T)
    i = np.arange(start, start + count, dtype=np.uint64)
    with np.errstate(over="ignore"):
        return i * D + (_stream(seed, start, count) % D)


def clustered_keys(T: int, seed: int = SEED_KEY, run: int = 1024) -> np.ndarray:
    """Sorted-run (clustered) keys: ceil(T/run) clusters of `run` consecutive integers."""
    if T == 0:
        return np.zeros(0, dtype=np.uint64)
    nc = (T + run - 1) // run
    Dc = ((1 << 64) - 2) // nc
    assert Dc > 2 * run
    c = np.arange(nc, dtype=np.uint64)
    with np.errstate(over="ignore"):
        base = c * np.uint64(Dc) + (_stream(seed ^ 0x5A5A, 0, nc) % np.uint64(Dc - run))
        keys = (base[:, None] + np.arange(run, dtype=np.uint64)[None, :]).reshape(-1)
    return np.ascontiguousarray(keys[:T])


def random_keys(T: int, seed: int = SEED_KEY, bits: int = 64) -> np.ndarray:
    """Truly random keys (sorted, de-duplicated, UINT64_MAX removed) for small tests."""
    rng = np.random.default_rng(seed & 0xFFFFFFFF)
    out = np.zeros(0, dtype=np.uint64)
    while out.shape[0] < T:
        x = rng.integers(0, 1 << 63, size=2 * T + 16, dtype=np.uint64, endpoint=False)
        x = (x << np.uint64(1)) | rng.integers(0, 2, size=x.shape[0], dtype=np.uint64)
        if bits < 64:
            x = x >> np.uint64(64 - bits)
        out = np.unique(np.concatenate([out, x[x != U64_MAX]]))
    if out.shape[0] > T:
        sel = np.sort(rng.choice(out.shape[0], size=T, replace=False))
        out = out[sel]
    return np.ascontiguousarray(out)


def values_for(keys: np.ndarray, seed: int = SEED_VAL) -> np.ndarray:
    """Key-derived values, so a routing or slot error shows up as a wrong value."""
    v = splitmix64(np.asarray(keys, dtype=np.uint64) ^ np.uint64(seed & _M64))
    v[v == U64_MAX] ^= np.uint64(1)
    return v


# ------------------------------------------------------------------------------ queries
def uniform_queries(keys: np.ndarray, Q: int, seed: int = SEED_QUERY, miss_frac: float = 0.0,
                    start: int = 0) -> np.ndarray:
    """Uniform over the key set (100 % hits); ``miss_frac`` of them replaced by random
    64-bit words (almost surely absent; the oracle decides)."""
    T = keys.shape[0]
    if T == 0:
        return _stream(seed ^ 0x77, start, Q)
    q = keys[_stream(seed, start, Q) % np.uint64(T)]
    if miss_frac > 0:
        sel = _unit(seed ^ 0x1111, start, Q) < miss_frac
        r = _stream(seed ^ 0x2222, start, Q)
        q = np.where(sel, r, q)
    return np.ascontiguousarray(q.astype(np.uint64))


@functools.lru_cache(maxsize=16)
def _zeta(n: int, theta: float) -> float:
    s = 0.0
    step = 1 << 22
    for b in range(1, n + 1, step):
        i = np.arange(b, min(n, b + step - 1) + 1, dtype=np.float64)
        s += float(np.sum(i ** (-theta)))
    return s


def zipf_ranks(n: int, Q: int, theta: float = 0.99, seed: int = SEED_QUERY, start: int = 0) -> np.ndarray:
    """Gray et al. / YCSB Zipfian rank generator over n items (rank 0 hottest)."""
    zetan = _zeta(n, theta)
    zeta2 = 1.0 + 0.5 ** theta
    alpha = 1.0 / (1.0 - theta)
    eta = (1.0 - (2.0 / n) ** (1.0 - theta)) / (1.0 - zeta2 / zetan)
    u = _unit(seed ^ 0x3333, start, Q)
    uz = u * zetan
    r = np.floor(n * (eta * u - eta + 1.0) ** alpha)
    r = np.where(uz < 1.0, 0.0, np.where(uz < 1.0 + 0.5 ** theta, 1.0, r))
    return np.minimum(r, n - 1).astype(np.uint64)


def zipf_queries(keys: np.ndarray, Q: int, theta: float = 0.99, seed: int = SEED_QUERY,
                 start: int = 0) -> np.ndarray:
    """ScrambledZipfian: rank -> key index by splitmix64(rank) mod T (hot keys scattered)."""
    T = keys.shape[0]
    ranks = zipf_ranks(T, Q, theta, seed, start)
    return np.ascontiguousarray(keys[splitmix64(ranks) % np.uint64(T)])


def sorted_run_queries(keys: np.ndarray, Q: int, run: int = 1024, seed: int = SEED_QUERY) -> np.ndarray:
    """Ascending runs of `run` consecutive keys from random start indices."""
    T = keys.shape[0]
    j = np.arange(Q, dtype=np.uint64)
    r = j // np.uint64(run)
    o = j % np.uint64(run)
    span = max(1, T - run + 1)
    st = splitmix64(np.uint64(seed ^ 0x4444) ^ r) % np.uint64(span)
    return np.ascontiguousarray(keys[(st + o) % np.uint64(T)])


def edge_queries(keys: np.ndarray) -> np.ndarray:
    """Boundary cases: 0, UINT64_MAX, first/last keys and their neighbours."""
    e = [0, 1, (1 << 64) - 1, (1 << 64) - 2, 1 << 63, (1 << 63) - 1]
    if keys.shape[0]:
        for k in (int(keys[0]), int(keys[-1]), int(keys[keys.shape[0] // 2])):
            e += [k, max(0, k - 1), min((1 << 64) - 1, k + 1)]
    return np.array(e, dtype=np.uint64)


# ------------------------------------------------------------------------------ ranges
def ranges(keys: np.ndarray, Qr: int, length: int, seed: int = SEED_RANGE):
    """lo = key[p], hi = key[p+len-1], p uniform in [0, T-len]  (count = len)."""
    T = keys.shape[0]
    span = max(1, T - length + 1)
    p = _stream(seed, 0, Qr) % np.uint64(span)
    hi_idx = np.minimum(p + np.uint64(length - 1), np.uint64(max(T - 1, 0)))
    return np.ascontiguousarray(keys[p]), np.ascontiguousarray(keys[hi_idx])


def random_ranges(keys: np.ndarray, Qr: int, seed: int = SEED_RANGE, max_width_keys: int = 64):
    """Mixed ranges for correctness: arbitrary 64-bit bounds (incl. lo > hi, empty gaps)."""
    T = keys.shape[0]
    a = _stream(seed ^ 0x55, 0, Qr)
    b = _stream(seed ^ 0x66, 0, Qr)
    kind = _stream(seed ^ 0x77, 0, Qr) % np.uint64(4)
    lo = a.copy()
    hi = b.copy()
    if T:
        p = a % np.uint64(T)
        w = b % np.uint64(max_width_keys)
        q = np.minimum(p + w, np.uint64(T - 1))
        lo = np.where(kind == 0, keys[p], lo)
        hi = np.where(kind == 0, keys[q], hi)
        lo = np.where(kind == 1, keys[p] - np.uint64(1), lo)            # may wrap for key 0: fine
        hi = np.where(kind == 1, keys[q] + np.uint64(1), hi)
    lo2 = np.minimum(lo, hi)
    hi2 = np.maximum(lo, hi)
    lo = np.where(kind == 3, hi2, np.where(kind == 2, lo, lo2))       # kind 3: lo > hi allowed
    hi = np.where(kind == 3, lo2, np.where(kind == 2, hi, hi2))
    return np.ascontiguousarray(lo.astype(np.uint64)), np.ascontiguousarray(hi.astype(np.uint64))


# ------------------------------------------------------------------------------ torch (device)
# The same counter-based streams computed with torch int64 tensors (wrapping arithmetic, bit
# patterns identical to the numpy uint64 versions) so that multi-GiB key sets and batches can
# be generated directly in device memory.  tests/test_gen.py pins them to the numpy versions.
def _t_lsr(x, s: int):
    import torch

    return (x >> s) & torch.tensor((1 << (64 - s)) - 1, dtype=torch.int64, device=x.device)


def _t_const(v: int, device):
    import torch

    return torch.tensor(v - (1 << 64) if v >= (1 << 63) else v, dtype=torch.int64, device=device)


def splitmix64_t(x):
    """splitmix64 over an int64 tensor holding uint64 bit patterns."""
    dev = x.device
    x = x + _t_const(0x9E3779B97F4A7C15, dev)
    z = (x ^ _t_lsr(x, 30)) * _t_const(0xBF58476D1CE4E5B9, dev)
    z = (z ^ _t_lsr(z, 27)) * _t_const(0x94D049BB133111EB, dev)
    return z ^ _t_lsr(z, 31)


def _t_umod(h, m: int):
    """unsigned 64-bit h mod m (m < 2^62) with int64 tensor ops."""
    half = _t_lsr(h, 1) % m
    return (half * 2 + (h & 1)) % m


def _t_stream(seed: int, start: int, n: int, device):
    import torch

    idx = torch.arange(start, start + n, dtype=torch.int64, device=device)
    return splitmix64_t(_t_const(seed & _M64, device) ^ idx)


def uniform_keys_t(T: int, device, seed: int = SEED_KEY, start: int = 0, count: int | None = None):
    """uniform_keys(T)[start:start+count] generated on `device` (int64 tensor of the uint64
    keys); a slice is e.g. one key-range shard of the partitioned configuration."""
    import torch

    if count is None:
        count = T - start
    D = ((1 << 64) - 2) // T
    i = torch.arange(start, start + count, dtype=torch.int64, device=device)
    return i * _t_const(D, device) + _t_umod(_t_stream(seed, start, count, device), D)


def values_for_t(keys, seed: int = SEED_VAL):
    v = splitmix64_t(keys ^ _t_const(seed & _M64, keys.device))
    return v ^ (v == -1).to(v.dtype)  # UINT64_MAX -> ^1


def uniform_queries_t(keys, Q: int, seed: int = SEED_QUERY, start: int = 0):
    T = keys.shape[0]
    return keys[_t_umod(_t_stream(seed, start, Q, keys.device), T)]


def keys_at_t(T: int, idx, seed: int = SEED_KEY):
    """uniform_keys(T)[idx] for an int64 index tensor (the closed form per index)."""
    D = ((1 << 64) - 2) // T
    return idx * _t_const(D, idx.device) + _t_umod(splitmix64_t(_t_const(seed & _M64, idx.device) ^ idx), D)


def _t_unit(seed: int, start: int, n: int, device):
    import torch

    return _t_lsr(_t_stream(seed, start, n, device), 11).to(torch.float64) * (1.0 / (1 << 53))


def zipf_queries_t(keys, Q: int, theta: float = 0.99, seed: int = SEED_QUERY, start: int = 0):
    """zipf_queries on the device (same streams and formulas in float64; equal to the numpy
    version up to the last-ulp rounding of pow, tests/test_gen.py)."""
    import torch

    T = keys.shape[0]
    zetan = _zeta(T, theta)
    zeta2 = 1.0 + 0.5 ** theta
    alpha = 1.0 / (1.0 - theta)
    eta = (1.0 - (2.0 / T) ** (1.0 - theta)) / (1.0 - zeta2 / zetan)
    u = _t_unit(seed ^ 0x3333, start, Q, keys.device)
    uz = u * zetan
    r = torch.floor(T * torch.pow(eta * u - eta + 1.0, alpha))
    r = torch.where(uz < 1.0, torch.zeros_like(r), torch.where(uz < 1.0 + 0.5 ** theta, torch.ones_like(r), r))
    r = torch.clamp(r, max=T - 1).to(torch.int64)
    return keys[_t_umod(splitmix64_t(r), T)]


def update_ops_t(T: int, n: int, insert_frac: float, delete_frac: float, device, seed: int = SEED_OPS,
                 lo: int = 0, hi: int | None = None):
    """update_ops over the keys uniform_keys(T)[lo:hi], generated on the device from indices
    (no key array needed: the partitioned config holds 2^29 keys per shard).  Inserts are the
    midpoints of random gaps, updates/deletes hit existing keys.  Returns (ops uint8, keys
    int64, values int64) tensors."""
    import torch

    hi = T if hi is None else hi
    u = _t_unit(seed, 0, n, device)
    span = max(1, hi - lo - 1)
    g = _t_umod(_t_stream(seed ^ 0x99, 0, n, device), span) + lo
    a, b = keys_at_t(T, g), keys_at_t(T, g + 1)
    mid = a + _t_lsr(b - a, 1)
    exist = keys_at_t(T, _t_umod(_t_stream(seed ^ 0x98, 0, n, device), hi - lo) + lo)
    is_ins = u < insert_frac
    is_del = (u >= insert_frac) & (u < insert_frac + delete_frac)
    k = torch.where(is_ins, mid, exist)
    ops = is_del.to(torch.uint8)
    v = values_for_t(_t_stream(seed ^ 0xAA, 0, n, device), seed ^ 0xBB)
    return ops, k, v


# ------------------------------------------------------------------------------ updates
def update_ops(keys: np.ndarray, n: int, insert_frac: float = 0.05, delete_frac: float = 0.0,
               seed: int = SEED_OPS):
    """A batch of n ops (5 % inserts + 95 % updates; config 5 adds 5 % deletes).

    op 0 = upsert, 1 = delete.  Inserts use fresh keys (midpoints of random gaps, or random
    words when the set is tiny); updates and deletes hit existing keys.
    Returns (ops uint8, keys uint64, values uint64)."""
    T = keys.shape[0]
    u = _unit(seed, 0, n)
    pick = _stream(seed ^ 0x99, 0, n)
    newv = values_for(_stream(seed ^ 0xAA, 0, n), seed ^ 0xBB)
    ops = np.zeros(n, dtype=np.uint8)
    out = np.empty(n, dtype=np.uint64)
    is_ins = u < insert_frac
    is_del = (u >= insert_frac) & (u < insert_frac + delete_frac)
    if T >= 2:
        g = pick % np.uint64(T - 1)
        a = keys[g]
        b = keys[g + np.uint64(1)]
        mid = a + (b - a) // np.uint64(2)
        fresh = np.where(b - a >= np.uint64(2), mid, _stream(seed ^ 0xCC, 0, n))
        exist = keys[pick % np.uint64(T)]
    else:
        fresh = _stream(seed ^ 0xCC, 0, n)
        exist = fresh
    fresh = np.where(fresh == U64_MAX, fresh - np.uint64(1), fresh)
    out[:] = np.where(is_ins, fresh, exist)
    ops[is_del] = 1
    return ops, out, newv
