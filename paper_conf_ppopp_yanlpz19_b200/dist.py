"""Multi-GPU Harmonia on one node: one process per GPU, torch.distributed for
the plumbing (NCCL over NVLink/NVSwitch on the GPU box, gloo in the CPU tests).

ReplicatedTree   every rank holds the same layout (built from the same seeded records); a
                 query batch is split 1/P per rank.  No collective on the hot path.
PartitionedTree  rank p owns the keys in [splitter[p-1], splitter[p]) (key quantiles) in its
                 own Harmonia layout.  Point queries: route (PSA partition by destination, the
                 C-ABI's harmonia_route_partition) -> all_to_all_single(counts) ->
                 all_to_all_single(queries) -> local search -> all_to_all_single(values, the
                 reverse splits) -> harmonia_scatter_results back to the caller's order.
                 Ranges are cut at every splitter they cross; pieces are answered by their
                 shards and concatenated in shard order (= key order).

The per-device steps go through a small `ops` object so that the exchange logic can be
tested on CPU with a gloo group (tests/test_dist.py injects CPU stand-ins); the default ops
are the CUDA kernels of libharmonia.so, and there is no CPU fallback on the product path.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from . import Tree, route_partition, scatter_results

__all__ = ["ReplicatedTree", "PartitionedTree", "CudaOps", "key_splitters"]


def _i64(t: torch.Tensor) -> torch.Tensor:
    """uint64 payloads travel as int64 (NCCL and gloo both move 8-byte words)."""
    return t.view(torch.int64) if t.dtype == torch.uint64 else t


def _u64(t: torch.Tensor) -> torch.Tensor:
    return t.view(torch.uint64) if t.dtype == torch.int64 else t


def _u64_words(values, device) -> torch.Tensor:
    """Python ints in [0, 2^64) as an int64 tensor holding the same 64-bit words."""
    import numpy as np

    a = np.asarray([int(v) for v in values], dtype=np.uint64).view(np.int64)
    return torch.from_numpy(a.copy()).to(device)


def key_splitters(sorted_keys, P: int):
    """Key-quantile splitters sigma_p = key[p*T/P], p = 1..P-1 (shard p owns [sigma_p, sigma_{p+1}))."""
    T = len(sorted_keys)
    return [int(sorted_keys[(p * T) // P]) for p in range(1, P)]


class CudaOps:
    """Device steps of the partitioned path, all in libharmonia.so kernels."""

    def __init__(self, tree: Tree, splitters: torch.Tensor, P: int):
        self.tree, self.split, self.P = tree, splitters, P

    def route(self, q):
        return route_partition(self.split, self.P, q)

    def search(self, q):
        return self.tree.search(q)

    def range(self, lo, hi, cap):
        return self.tree.range(lo, hi, cap)

    def scatter(self, vals, pos):
        return scatter_results(vals, pos)


class ReplicatedTree:
    """Same layout on every rank; each rank answers its own slice of the global batch."""

    def __init__(self, keys, values, fanout: int = 64, fill: float = 1.0, group=None):
        self.group = group
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        self.tree = Tree(keys, values, fanout=fanout, fill=fill)

    def slice_of(self, n_global: int):
        """[begin, end) of this rank's share of an n_global-query batch."""
        b = (n_global * self.rank) // self.world
        return b, (n_global * (self.rank + 1)) // self.world

    def search(self, q_local, **kw):
        return self.tree.search(q_local, **kw)

    def range(self, lo, hi, cap, **kw):
        return self.tree.range(lo, hi, cap, **kw)


class PartitionedTree:
    """Key-range partitioned layout: this rank's shard plus the global splitters."""

    def __init__(self, local_keys, local_values, splitters, fanout: int = 64, fill: float = 1.0, group=None,
                 ops=None, device=None):
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        assert len(splitters) == self.world - 1, "P-1 splitters for P ranks"
        if ops is None:
            dev = device if device is not None else torch.device("cuda", torch.cuda.current_device())
            tree = Tree(local_keys, local_values, fanout=fanout, fill=fill, device=dev)
            ops = CudaOps(tree, _u64_words(splitters, dev).view(torch.uint64), self.world)
        self.ops = ops
        self.splitters = list(splitters)

    # ------------------------------------------------------------------ point queries
    def search(self, q: torch.Tensor) -> torch.Tensor:
        P = self.world
        routed, pos, counts = self.ops.route(q)              # destination-major grouping
        dev = q.device
        send = torch.tensor(counts, dtype=torch.int64, device=dev)
        recv = torch.empty(P, dtype=torch.int64, device=dev)
        dist.all_to_all_single(recv, send, group=self.group)  # C3: destination counts
        rc = recv.tolist()
        recv_q = torch.empty(sum(rc), dtype=torch.int64, device=dev)
        dist.all_to_all_single(recv_q, _i64(routed), output_split_sizes=rc, input_split_sizes=counts,
                               group=self.group)               # C4: route queries
        vals = self.ops.search(_u64(recv_q))                   # local Harmonia search
        back = torch.empty(q.numel(), dtype=torch.int64, device=dev)
        dist.all_to_all_single(back, _i64(vals), output_split_sizes=counts, input_split_sizes=rc,
                               group=self.group)               # C5: return values
        return self.ops.scatter(_u64(back), pos)               # caller's order

    # ------------------------------------------------------------------ range queries
    def range(self, lo: torch.Tensor, hi: torch.Tensor, cap: int):
        """Inclusive ranges; a range crossing splitters is answered piecewise by every shard it
        touches; pieces are concatenated in shard order (= key order) and the slab is cut at
        `cap`.  Returns (keys [n, cap] uint64, values [n, cap] uint64, counts [n] int64 = true
        totals); slab entries past the count hold PAD / NOT_FOUND."""
        P, dev, n = self.world, lo.device, lo.numel()
        sign = torch.tensor(-(1 << 63), dtype=torch.int64, device=dev)
        ulo, uhi = _i64(lo) ^ sign, _i64(hi) ^ sign          # unsigned order as signed order
        spi = _u64_words(self.splitters, dev)
        if P > 1:
            d_lo = torch.searchsorted(spi ^ sign, ulo, right=True)
            d_hi = torch.searchsorted(spi ^ sign, uhi, right=True)
        else:
            d_lo = d_hi = torch.zeros(n, dtype=torch.int64, device=dev)
        npieces = torch.where(ulo > uhi, torch.ones_like(d_lo), d_hi - d_lo + 1)
        first_of_q = torch.cumsum(npieces, 0) - npieces
        qid = torch.repeat_interleave(torch.arange(n, device=dev), npieces)
        off = torch.arange(qid.numel(), device=dev) - first_of_q[qid]
        shard = d_lo[qid] + off
        plo, phi = _i64(lo)[qid].clone(), _i64(hi)[qid].clone()
        if P > 1:
            first = off > 0
            plo[first] = spi[shard[first] - 1]
            last = off < (npieces[qid] - 1)
            phi[last] = spi[shard[last]] - 1                # splitter keys belong to the upper shard
        order = torch.argsort(shard, stable=True)
        counts = torch.bincount(shard, minlength=P)
        send_n = counts.tolist()
        recv_counts = torch.empty(P, dtype=torch.int64, device=dev)
        dist.all_to_all_single(recv_counts, counts.to(torch.int64), group=self.group)
        rc = recv_counts.tolist()
        pieces = torch.stack([plo[order], phi[order]], 1).contiguous()
        recv_p = torch.empty(sum(rc), 2, dtype=torch.int64, device=dev)
        dist.all_to_all_single(recv_p, pieces, output_split_sizes=rc, input_split_sizes=send_n, group=self.group)
        m = recv_p.shape[0]
        ko, vo, cnt = self.ops.range(_u64(recv_p[:, 0].contiguous()), _u64(recv_p[:, 1].contiguous()), cap)
        cols = [cnt.to(torch.int64).reshape(m, 1)]
        if cap:
            cols = [_i64(ko).reshape(m, cap), _i64(vo).reshape(m, cap)] + cols
        payload = torch.cat(cols, 1).contiguous()
        back = torch.empty(qid.numel(), payload.shape[1], dtype=torch.int64, device=dev)
        dist.all_to_all_single(back, payload, output_split_sizes=send_n, input_split_sizes=rc, group=self.group)
        res = torch.empty_like(back)
        res[order] = back                                     # pieces back in (query, shard) order
        pc = res[:, -1]
        total = torch.zeros(n, dtype=torch.int64, device=dev).index_add_(0, qid, pc)
        out_k = torch.full((n, cap), -1, dtype=torch.int64, device=dev)
        out_v = torch.full((n, cap), -1, dtype=torch.int64, device=dev)
        if cap:
            S = torch.cumsum(pc, 0) - pc
            before = S - S[first_of_q[qid]]                   # records of earlier pieces of the query
            t = torch.arange(cap, device=dev)
            slot = before[:, None] + t[None, :]
            valid = (t[None, :] < torch.clamp(pc, max=cap)[:, None]) & (slot < cap)
            rows = qid[:, None].expand(-1, cap)[valid]
            out_k[rows, slot[valid]] = res[:, :cap][valid]
            out_v[rows, slot[valid]] = res[:, cap:2 * cap][valid]
        return _u64(out_k), _u64(out_v), total
