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
PeerPartitionedTree  the same shards with the exchange fused into the kernels over peer memory
                 (no NCCL data collective): harmonia_route_count -> all_gather of the P x P count
                 matrix -> harmonia_route_push writes every destination's run straight into
                 that rank's receive buffer (CUDA IPC mapping, NVLink stores) -> device
                 barrier -> local search of the receive buffer -> harmonia_segments_push
                 returns every source's results into its "back" buffer -> device barrier ->
                 harmonia_route_return (inverse partition) restores the caller's order.  The
                 barriers are harmonia_peer_barrier kernels (flags in peer memory, system-scope
                 release/acquire): the only host wait per batch is the count matrix.

The per-device steps go through a small `ops` object so that the exchange logic can be
tested on CPU with a gloo group (tests/test_dist.py injects CPU stand-ins); the default ops
are the CUDA kernels of libharmonia.so, and there is no CPU fallback on the product path.
"""
from __future__ import annotations

import torch
import torch.distributed as dist

from . import (HarmoniaError, Tree, range_assemble, range_split, route_partition, route_update_payload,
               scatter_results, update_validate)

__all__ = ["ReplicatedTree", "PartitionedTree", "PeerPartitionedTree", "CudaOps", "CudaPeerOps", "key_splitters",
           "peer_offsets"]


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

    def validate_update(self, ops, keys, values):
        return update_validate(ops, keys, values)

    def route_update(self, ops, keys, values, rank: int):
        rk, pos, counts = route_partition(self.split, self.P, keys)
        ro, rv, rs = route_update_payload(ops, values, pos, rank)
        return rk, ro, rv, rs, counts

    def update(self, ops, keys, values, seq):
        self.tree.update(ops, keys, values, seq=seq)

    def range_split(self, lo, hi):
        return range_split(self.split, self.P, lo, hi)

    def range_assemble(self, n, cap, pbase, pid, counts, keys, values):
        return range_assemble(n, cap, pbase, pid, counts, keys, values)


def _routed_update(tree_like, ops, keys, values):
    """Batched updates on a key-range partitioned tree (updates are routed like
    queries).  Each op goes to the shard owning its key, with its global sequence number
    rank << 32 | position, so a shard applies the ops it receives in the global batch order
    (rank-major, then each rank's batch order; C-A18 last-op-wins) whatever order routing
    and the exchange deliver them in.  Collective: every rank calls it (possibly with 0 ops)."""
    ops_ = tree_like.ops
    group, P = tree_like.group, tree_like.world
    if P == 1:  # one shard: the batch applies in place, in batch order (C-A18)
        ops_.update(ops, keys, values, None)
        return
    # all shards accept the batch or all reject it: every rank's ops are validated before any
    # is routed, the verdict is all-reduced, and every rank raises the same error
    flag = ops_.validate_update(ops, keys, values).to(torch.int32)
    dist.all_reduce(flag, op=dist.ReduceOp.MAX, group=group)
    bad = int(flag.item())
    if bad:
        raise HarmoniaError(3 if bad & 2 else 1, "partitioned update (some rank's batch)")
    rk, ro, rv, rs, counts = ops_.route_update(ops, keys, values, tree_like.rank)
    dev = keys.device
    send = torch.tensor(counts, dtype=torch.int64, device=dev)
    recv = torch.empty(P, dtype=torch.int64, device=dev)
    dist.all_to_all_single(recv, send, group=group)
    rc = recv.tolist()
    m = sum(rc)

    def a2a(x, dtype):
        out = torch.empty(m, dtype=dtype, device=dev)
        dist.all_to_all_single(out, x, output_split_sizes=rc, input_split_sizes=counts, group=group)
        return out

    k = a2a(_i64(rk), torch.int64)
    v = a2a(_i64(rv), torch.int64)
    sq = a2a(_i64(rs), torch.int64)
    o = a2a(ro, torch.uint8)
    if m:
        ops_.update(o, _u64(k), _u64(v), _u64(sq))


class ReplicatedTree:
    """Same layout on every rank; each rank answers its own slice of the global batch."""

    def __init__(self, keys, values, fanout: int = 64, fill: float = 1.0, group=None, tree=None):
        self.group = group
        self.rank = dist.get_rank(group) if dist.is_initialized() else 0
        self.world = dist.get_world_size(group) if dist.is_initialized() else 1
        # `tree`: any object with search/range (tests inject a CPU stand-in); default: the layout
        # on this rank's device, built from the same seeded records on every rank
        self.tree = tree if tree is not None else Tree(keys, values, fanout=fanout, fill=fill)

    def slice_of(self, n_global: int):
        """[begin, end) of this rank's share of an n_global-query batch."""
        b = (n_global * self.rank) // self.world
        return b, (n_global * (self.rank + 1)) // self.world

    def search(self, q_local, **kw):
        return self.tree.search(q_local, **kw)

    def search_global(self, q_global, gather: bool = False, **kw):
        """This rank answers its slice of a batch every rank holds; no collective on the hot
        path.  gather=True all-gathers the slices into the full result (outside any timed
        region: it is the only collective of this mode)."""
        b, e = self.slice_of(q_global.numel())
        mine = self.search(q_global[b:e], **kw)
        if not gather or self.world == 1:
            return mine
        n = q_global.numel()
        parts = [torch.empty((n * (r + 1)) // self.world - (n * r) // self.world, dtype=torch.int64,
                             device=mine.device) for r in range(self.world)]
        dist.all_gather(parts, _i64(mine).contiguous(), group=self.group)
        return _u64(torch.cat(parts))

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
    def search(self, q: torch.Tensor, slices: int = 1) -> torch.Tensor:
        """Point queries routed to their shards.  slices > 1 splits the batch so that the
        exchange of slice i+1 overlaps the local search of slice i: every
        slice is routed on the caller's stream, its query all-to-all is asynchronous, the
        search runs on a side stream once the exchange has landed, and the results go back
        slice by slice (collectives are issued in the same order on every rank)."""
        P = self.world
        if P == 1:  # one shard: nothing to route (no partition pass, no exchange, no scatter)
            return self.ops.search(q)
        if slices > 1 and q.numel() >= slices:
            return self._search_sliced(q, slices)
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

    def search_host(self, q_host: torch.Tensor, out_host: torch.Tensor, **kw) -> torch.Tensor:
        """Point queries from and to pinned host memory.  One shard: the tree's own three-stage
        host pipeline (harmonia_search_batch_host, H2D / search / D2H overlapped chunk by
        chunk); several shards: one H2D copy, the routed search, one D2H copy."""
        if self.world == 1 and hasattr(self.ops, "tree"):
            return self.ops.tree.search_host(q_host, out_host, **kw)
        dev = self.ops.tree.device if hasattr(self.ops, "tree") else q_host.device
        q = q_host.to(dev, non_blocking=True)
        out_host.copy_(self.search(q), non_blocking=True)
        return out_host

    def _search_sliced(self, q, slices):
        import contextlib

        dev = q.device
        cuda = dev.type == "cuda"
        side = torch.cuda.Stream(dev) if cuda else None
        main = torch.cuda.current_stream(dev) if cuda else None
        n = q.numel()
        cuts = [(n * i) // slices for i in range(slices + 1)]
        pending = []  # (recv handle, recv buffer, counts, rc, pos, lo, hi)
        for i in range(slices):  # route + exchange every slice; searches start as exchanges land
            qs = q[cuts[i]:cuts[i + 1]]
            routed, pos, counts = self.ops.route(qs)
            send = torch.tensor(counts, dtype=torch.int64, device=dev)
            recv = torch.empty(self.world, dtype=torch.int64, device=dev)
            dist.all_to_all_single(recv, send, group=self.group)
            rc = recv.tolist()
            recv_q = torch.empty(sum(rc), dtype=torch.int64, device=dev)
            work = dist.all_to_all_single(recv_q, _i64(routed), output_split_sizes=rc, input_split_sizes=counts,
                                          group=self.group, async_op=True)
            pending.append((work, recv_q, counts, rc, pos, cuts[i], cuts[i + 1], routed))
        out = torch.empty(n, dtype=q.dtype, device=dev)
        results = []
        for work, recv_q, counts, rc, pos, lo, hi, routed in pending:
            with (torch.cuda.stream(side) if cuda else contextlib.nullcontext()):
                work.wait()                                    # this slice's queries have landed
                vals = self.ops.search(_u64(recv_q))
                ev = torch.cuda.Event() if cuda else None
                if cuda:
                    ev.record(side)
                    recv_q.record_stream(side)
            results.append((vals, ev, counts, rc, pos, lo, hi))
        for vals, ev, counts, rc, pos, lo, hi in results:
            if cuda:
                main.wait_event(ev)
                vals.record_stream(main)
            back = torch.empty(hi - lo, dtype=torch.int64, device=dev)
            dist.all_to_all_single(back, _i64(vals), output_split_sizes=counts, input_split_sizes=rc,
                                   group=self.group)
            out[lo:hi] = self.ops.scatter(_u64(back), pos)
        return out

    # ------------------------------------------------------------------ updates
    def update(self, ops, keys, values):
        """Batched upsert (op 0) / delete (op 1) routed to the owning shards (collective)."""
        _routed_update(self, ops, keys, values)

    # ------------------------------------------------------------------ range queries
    def range(self, lo: torch.Tensor, hi: torch.Tensor, cap: int):
        """Inclusive ranges; a range crossing splitters is answered piecewise by every shard it
        touches (harmonia_range_split_*), pieces are concatenated in shard order (= key order)
        and the slab is cut at `cap` (harmonia_range_assemble).  Returns (keys [n, cap] uint64,
        values [n, cap] uint64, counts [n] = true totals); slab entries past the count hold
        PAD / NOT_FOUND."""
        n, dev = lo.numel(), lo.device
        if self.world == 1:
            return self.ops.range(lo, hi, cap)
        plo, phi, pid, send_n, pbase = self.ops.range_split(lo, hi)   # kernels: cut + dest-major
        recv_counts = torch.empty(self.world, dtype=torch.int64, device=dev)
        dist.all_to_all_single(recv_counts, torch.tensor(send_n, dtype=torch.int64, device=dev), group=self.group)
        rc = recv_counts.tolist()
        pieces = torch.stack([_i64(plo), _i64(phi)], 1).contiguous()
        recv_p = torch.empty(sum(rc), 2, dtype=torch.int64, device=dev)
        dist.all_to_all_single(recv_p, pieces, output_split_sizes=rc, input_split_sizes=send_n, group=self.group)
        m = recv_p.shape[0]
        ko, vo, cnt = self.ops.range(_u64(recv_p[:, 0].contiguous()), _u64(recv_p[:, 1].contiguous()), cap)
        cols = [cnt.to(torch.int64).reshape(m, 1)]
        if cap:
            cols = [_i64(ko).reshape(m, cap), _i64(vo).reshape(m, cap)] + cols
        payload = torch.cat(cols, 1).contiguous()
        back = torch.empty(plo.numel(), payload.shape[1], dtype=torch.int64, device=dev)
        dist.all_to_all_single(back, payload, output_split_sizes=send_n, input_split_sizes=rc, group=self.group)
        bc = back[:, -1].to(torch.int32).contiguous()
        bk = _u64(back[:, :cap].contiguous()) if cap else None
        bv = _u64(back[:, cap:2 * cap].contiguous()) if cap else None
        return self.ops.range_assemble(n, cap, pbase, pid, bc, bk, bv)   # kernel: shard order, cap


# ------------------------------------------------------------------ fused routing (peer memory)
def peer_offsets(M, me: int):
    """Offsets of the peer exchange from the P x P count matrix M[p][d] (queries rank p routes
    to shard d), for rank `me`:
      push_off[d]  element offset of me's run in d's receive buffer   = sum_{p<me} M[p][d]
      recv_off[p]  where source p's segment starts in me's receive buffer = sum_{p'<p} M[p'][me]
      recv_n       queries me receives                               = sum_p M[p][me]
      back_off[p]  offset of me's run in p's routed order (= in p's back buffer) = sum_{d<me} M[p][d]
    """
    P = len(M)
    push_off = [sum(M[p][d] for p in range(me)) for d in range(P)]
    recv_off = [sum(M[q][me] for q in range(p)) for p in range(P)]
    recv_n = sum(M[p][me] for p in range(P))
    back_off = [sum(M[p][d] for d in range(me)) for p in range(P)]
    return push_off, recv_off, recv_n, back_off


class CudaPeerOps:
    """Device steps and peer buffers of PeerPartitionedTree (libharmonia.so kernels, CUDA IPC)."""

    def __init__(self, tree: Tree, splitters: torch.Tensor, P: int, group=None, device_barrier: bool = True):
        self.tree, self.split, self.P, self.group = tree, splitters, P, group
        self.dev = tree.device
        self.recv = self.back = None
        self.recv_addr, self.back_addr = [], []
        self.cap_recv = self.cap_back = 0
        self.ws, self.ws_n = None, -1
        self.device_barrier = device_barrier
        self.flags = None           # this rank's flag array (PeerBuffer, P uint64)
        self.flag_addrs = None      # device uint64[P]: every rank's flag array, mapped here
        self.flag_maps = []
        self.epoch = 0
        self.err = None

    # buffers --------------------------------------------------------------------------
    def ensure_capacity(self, cap_recv: int, cap_back: int):
        """Collective: every rank calls it with the same (cap_recv, cap_back)."""
        from . import PeerBuffer

        if cap_recv <= self.cap_recv and cap_back <= self.cap_back:
            return
        self.close()
        cap_recv, cap_back = max(cap_recv, 1), max(cap_back, 1)
        self.recv, self.back = PeerBuffer(cap_recv * 8), PeerBuffer(cap_back * 8)
        mine = (self.recv.handle_bytes(), self.back.handle_bytes())
        allh = [None] * self.P
        dist.all_gather_object(allh, mine, group=self.group)
        me = dist.get_rank(self.group)
        self.recv_addr = [self.recv.addr if p == me else PeerBuffer.open(allh[p][0]) for p in range(self.P)]
        self.back_addr = [self.back.addr if p == me else PeerBuffer.open(allh[p][1]) for p in range(self.P)]
        self.cap_recv, self.cap_back = cap_recv, cap_back
        if self.device_barrier and self.flags is None:  # once: flags outlive buffer growth
            self.flags = PeerBuffer(8 * self.P)
            allf = [None] * self.P
            dist.all_gather_object(allf, self.flags.handle_bytes(), group=self.group)
            addrs = [self.flags.addr if p == me else PeerBuffer.open(allf[p]) for p in range(self.P)]
            self.flag_maps = [a for p, a in enumerate(addrs) if p != me]
            self.flag_addrs = torch.tensor([a - (1 << 64) if a >= (1 << 63) else a for a in addrs],
                                           dtype=torch.int64, device=self.dev)
            self.err = torch.zeros(1, dtype=torch.int32, device=self.dev)

    def check(self):
        """Raise if a device barrier timed out (reads one flag; the caller has synchronised)."""
        if self.err is not None and int(self.err.item()):
            raise HarmoniaError(5, "harmonia_peer_barrier: timed out waiting for a peer")

    def close(self):
        from . import PeerBuffer

        if self.recv is None:
            return
        torch.cuda.synchronize(self.dev)
        dist.barrier(group=self.group)  # no peer still writes into the buffers being released
        me = dist.get_rank(self.group)
        for p in range(self.P):
            if p != me:
                PeerBuffer.close_mapping(self.recv_addr[p])
                PeerBuffer.close_mapping(self.back_addr[p])
        for a in self.flag_maps:
            PeerBuffer.close_mapping(a)
        dist.barrier(group=self.group)  # every mapping closed before the owners free
        self.recv.free()
        self.back.free()
        if self.flags is not None:
            self.flags.free()
        self.recv = self.back = self.flags = None
        self.flag_maps, self.flag_addrs = [], None
        self.cap_recv = self.cap_back = 0

    # steps ----------------------------------------------------------------------------
    def route_count(self, q):
        from . import route_count, route_workspace

        n = q.numel()
        if self.ws is None or n > self.ws_n:
            self.ws, self.ws_n = route_workspace(self.P, max(n, 1), self.dev), n
        return route_count(self.split, self.P, q, self.ws)

    def route_push(self, q, targets):
        from . import route_push

        route_push(self.split, self.P, q, [self.recv_addr[d] + 8 * off for d, off in targets], self.ws)

    def search_recv(self, n: int):
        out = torch.empty(n, dtype=torch.uint64, device=self.dev)
        if n:
            self.tree.search_addr(self.recv.addr, n, out)
        return out

    def segments_push(self, vals, segs):
        from . import segments_push

        segs = [s for s in segs if s[1] > 0]
        if segs:
            segments_push(vals, [s[0] for s in segs], [s[1] for s in segs],
                          [self.back_addr[s[2]] + 8 * s[3] for s in segs], self.ws)

    def route_return(self, n: int):
        from . import route_return

        out = torch.empty(n, dtype=torch.uint64, device=self.dev)
        if n:
            route_return(self.P, self.back.addr, n, out, self.ws)
        return out

    def fence(self):
        torch.cuda.current_stream(self.dev).synchronize()  # the pushes of this rank are complete

    def barrier(self):
        """Every rank's pushes so far are visible to the work queued after this on the stream."""
        if not self.device_barrier:
            self.fence()
            dist.barrier(group=self.group)
            return
        from . import peer_barrier

        self.epoch += 1
        peer_barrier(self.P, dist.get_rank(self.group), self.flag_addrs, self.flags.addr, self.epoch, self.err)

    def route_update(self, ops, keys, values, rank: int):
        rk, pos, counts = route_partition(self.split, self.P, keys)
        ro, rv, rs = route_update_payload(ops, values, pos, rank)
        return rk, ro, rv, rs, counts

    def update(self, ops, keys, values, seq):
        self.tree.update(ops, keys, values, seq=seq)


class PeerPartitionedTree:
    """Key-range partitioned layout whose query exchange runs over peer memory (no NCCL data
    collective): the route kernel stores every query straight into its shard's receive
    buffer and the results come back the same way."""

    def __init__(self, local_keys, local_values, splitters, fanout: int = 64, fill: float = 1.0, group=None,
                 ops=None, device=None, device_barrier: bool = True):
        self.group = group
        self.rank = dist.get_rank(group)
        self.world = dist.get_world_size(group)
        assert len(splitters) == self.world - 1, "P-1 splitters for P ranks"
        if ops is None:
            dev = device if device is not None else torch.device("cuda", torch.cuda.current_device())
            tree = Tree(local_keys, local_values, fanout=fanout, fill=fill, device=dev)
            ops = CudaPeerOps(tree, _u64_words(splitters, dev).view(torch.uint64), self.world, group,
                              device_barrier=device_barrier)
        self.ops = ops
        self.splitters = list(splitters)

    def _count_matrix(self, counts):
        nccl = dist.get_backend(self.group) == "nccl"
        dev = torch.device("cuda", torch.cuda.current_device()) if nccl else torch.device("cpu")
        mine = torch.tensor(counts, dtype=torch.int64, device=dev)
        allc = torch.empty(self.world * self.world, dtype=torch.int64, device=dev)
        dist.all_gather_into_tensor(allc, mine, group=self.group)
        a = allc.view(self.world, self.world).tolist()
        return a

    def search(self, q: torch.Tensor) -> torch.Tensor:
        P, me, n = self.world, self.rank, q.numel()
        counts = self.ops.route_count(q)                       # kernel: destination ranks
        M = self._count_matrix(counts)                         # P x P ints (the host wait)
        if hasattr(self.ops, "check"):
            self.ops.check()                                   # the previous batch's barriers
        push_off, recv_off, recv_n, back_off = peer_offsets(M, me)
        need_recv = max(sum(M[p][d] for p in range(P)) for d in range(P))
        need_back = max(sum(row) for row in M)
        self.ops.ensure_capacity(need_recv, need_back)         # collective, same numbers everywhere
        self.ops.route_push(q, [(d, push_off[d]) for d in range(P)])  # kernel: NVLink stores
        self._barrier()                                        # every run has arrived
        vals = self.ops.search_recv(recv_n)                    # local Harmonia search
        self.ops.segments_push(vals, [(recv_off[p], M[p][me], p, back_off[p]) for p in range(P)])
        self._barrier()                                        # every result has arrived
        return self.ops.route_return(n)                        # kernel: caller's order

    def _barrier(self):
        if hasattr(self.ops, "barrier"):
            self.ops.barrier()                                 # device-side (peer-memory flags)
        else:
            self.ops.fence()
            dist.barrier(group=self.group)

    def update(self, ops, keys, values):
        """Batched upsert (op 0) / delete (op 1) routed to the owning shards (collective)."""
        _routed_update(self, ops, keys, values)

    def close(self):
        if hasattr(self.ops, "check"):
            torch.cuda.synchronize()
            self.ops.check()
        if hasattr(self.ops, "close"):
            self.ops.close()
