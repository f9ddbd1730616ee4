"""Multi-process (gloo, world_size 2 and 3) tests of the partitioned-mode exchange logic.

The device steps (route / local search / local range / scatter back) are replaced by CPU
stand-ins built on the oracle, so these tests check the host-side routing, splits, the
all_to_all exchanges and the reassembly of points and multi-shard ranges against the oracle
over the *global* key set.  The CUDA ops themselves are checked in tests/test_gpu_*.py."""
import os
import socket

import numpy as np
import pytest
import torch
import torch.distributed as dist
import torch.multiprocessing as mp

import harmonia_gen as gen


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


class CpuOps:
    """Oracle-backed stand-ins for the CUDA steps of PartitionedTree (test only)."""

    def __init__(self, keys, vals, splitters, P):
        import oracle

        self.orc, self.keys, self.vals = oracle, keys, vals
        self.split = np.asarray(splitters, dtype=np.uint64)
        self.P = P

    def route(self, q):
        qn = q.view(torch.int64).numpy().view(np.uint64)
        dest = np.searchsorted(self.split, qn, side="right")
        pos = np.argsort(dest, kind="stable")
        counts = np.bincount(dest, minlength=self.P).tolist()
        return (torch.from_numpy(qn[pos].view(np.int64).copy()).view(torch.uint64),
                torch.from_numpy(pos.astype(np.int64)), counts)

    def search(self, q):
        qn = q.view(torch.int64).numpy().view(np.uint64)
        out = self.orc.sorted_search(self.keys, self.vals, qn, 1)
        return torch.from_numpy(out.view(np.int64).copy()).view(torch.uint64)

    def range(self, lo, hi, cap):
        ko, vo, cnt = self.orc.sorted_range(self.keys, self.vals, lo.view(torch.int64).numpy().view(np.uint64),
                                            hi.view(torch.int64).numpy().view(np.uint64), cap, 1)
        m = lo.numel()
        if cap:  # untouched slab entries are unspecified; make them PAD like the CUDA path
            mask = np.arange(cap)[None, :] >= np.minimum(cnt.astype(np.int64), cap)[:, None]
            ko = ko.reshape(m, cap).copy()
            vo = vo.reshape(m, cap).copy()
            ko[mask] = np.uint64(0xFFFFFFFFFFFFFFFF)
            vo[mask] = np.uint64(0xFFFFFFFFFFFFFFFF)
        t = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int64).copy()).view(torch.uint64)
        return (t(ko) if cap else None), (t(vo) if cap else None), torch.from_numpy(cnt.astype(np.int64))

    def scatter(self, vals, pos):
        out = torch.empty_like(vals.view(torch.int64))
        out[pos] = vals.view(torch.int64)
        return out.view(torch.uint64)

    def range_split(self, lo, hi):
        # cut at the splitters (the semantics of harmonia_range_split_*), destination-major,
        # and deliberately scrambled inside each destination's run (the kernel's order is
        # unspecified; the piece ids carry the order)
        l = lo.view(torch.int64).numpy().view(np.uint64)
        h = hi.view(torch.int64).numpy().view(np.uint64)
        d0 = np.searchsorted(self.split, l, side="right")
        np_ = np.where(l > h, 1, np.searchsorted(self.split, h, side="right") - d0 + 1)
        pbase = np.concatenate([[0], np.cumsum(np_)]).astype(np.uint32)
        plo, phi, dest, pid = [], [], [], []
        for i in range(len(l)):
            for j in range(int(np_[i])):
                d = int(d0[i]) + j
                a, b = l[i], h[i]
                if l[i] <= h[i]:
                    if j > 0:
                        a = self.split[d - 1]
                    if j + 1 < np_[i]:
                        b = self.split[d] - np.uint64(1)
                plo.append(a), phi.append(b), dest.append(d), pid.append(pbase[i] + j)
        dest = np.asarray(dest, dtype=np.int64)
        order = np.lexsort((-np.arange(len(dest)), dest))
        t = lambda a, dt: torch.from_numpy(np.asarray(a, dtype=dt)[order].copy())
        return (t(plo, np.uint64).view(torch.int64).view(torch.uint64), t(phi, np.uint64).view(torch.int64).view(torch.uint64),
                t(pid, np.uint32).to(torch.int64), np.bincount(dest, minlength=self.P).tolist(), torch.from_numpy(pbase))

    def range_assemble(self, n, cap, pbase, pid, counts, keys, values):
        pb, pid = pbase.numpy(), pid.numpy()
        row_of = np.empty(len(pid), dtype=np.int64)
        row_of[pid] = np.arange(len(pid))
        c = counts.numpy().astype(np.int64)
        k = keys.view(torch.int64).numpy().reshape(-1, cap) if cap else None
        v = values.view(torch.int64).numpy().reshape(-1, cap) if cap else None
        ko = np.full((n, cap), -1, dtype=np.int64)
        vo = np.full((n, cap), -1, dtype=np.int64)
        tot = np.zeros(n, dtype=np.int64)
        for i in range(n):
            f = 0
            for p in range(pb[i], pb[i + 1]):
                r = row_of[p]
                tot[i] += c[r]
                take = min(c[r], cap - f) if f < cap else 0
                if take:
                    ko[i, f:f + take] = k[r, :take]
                    vo[i, f:f + take] = v[r, :take]
                f += take
        return torch.from_numpy(ko).view(torch.uint64), torch.from_numpy(vo).view(torch.uint64), torch.from_numpy(tot)

    def validate_update(self, ops, keys, values):
        kn = keys.view(torch.int64).numpy().view(np.uint64)
        vn = values.view(torch.int64).numpy().view(np.uint64)
        o = ops.numpy()
        pad = np.uint64(0xFFFFFFFFFFFFFFFF)
        bad = (2 if bool(np.any(kn == pad) or np.any((o == 0) & (vn == pad))) else 0) | (4 if bool(np.any(o > 1)) else 0)
        return torch.tensor([bad], dtype=torch.int32)

    def route_update(self, ops, keys, values, rank):
        kn = keys.view(torch.int64).numpy().view(np.uint64)
        dest = np.searchsorted(self.split, kn, side="right")
        pos = np.argsort(dest, kind="stable")[::-1].copy()  # any order: the seq numbers carry it
        pos = pos[np.argsort(dest[pos], kind="stable")]
        t = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int64).copy())
        seq = (np.uint64(rank) << np.uint64(32)) | pos.astype(np.uint64)
        return (t(kn[pos]).view(torch.uint64), torch.from_numpy(ops.numpy()[pos].copy()),
                t(values.view(torch.int64).numpy().view(np.uint64)[pos]).view(torch.uint64), t(seq).view(torch.uint64),
                np.bincount(dest, minlength=self.P).tolist())

    def update(self, ops, keys, values, seq):
        order = (np.arange(keys.numel()) if seq is None
                 else np.argsort(seq.view(torch.int64).numpy().view(np.uint64), kind="stable"))
        m = self.orc.UpdateMap(self.keys, self.vals)
        m.apply(ops.numpy()[order], keys.view(torch.int64).numpy().view(np.uint64)[order],
                values.view(torch.int64).numpy().view(np.uint64)[order])
        self.keys, self.vals = m.dump()


def _worker(rank, world, port, T, cap, result_q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_ppopp_yanlpz19_b200.dist import PartitionedTree, key_splitters

        keys = gen.uniform_keys(T)
        vals = gen.values_for(keys)
        sp = key_splitters(keys, world)
        bounds = [0] + [int(np.searchsorted(keys, np.uint64(s))) for s in sp] + [T]
        lk, lv = keys[bounds[rank]:bounds[rank + 1]], vals[bounds[rank]:bounds[rank + 1]]
        ops = CpuOps(lk, lv, sp, world)
        pt = PartitionedTree(lk, lv, sp, ops=ops)
        # point queries: hits, misses, edges, splitter keys themselves
        q = np.concatenate([gen.uniform_queries(keys, 3000 + 17 * rank, seed=gen.SEED_QUERY + rank, miss_frac=0.3),
                            gen.edge_queries(keys), np.asarray(sp, dtype=np.uint64),
                            np.asarray(sp, dtype=np.uint64) - np.uint64(1)])
        qt = torch.from_numpy(q.view(np.int64).copy()).view(torch.uint64)
        got = pt.search(qt).view(torch.int64).numpy().view(np.uint64)
        exp = oracle.sorted_search(keys, vals, q)
        ok_pts = bool(np.array_equal(got, exp))
        # the sliced exchange (slice i+1 in flight while slice i is searched) gives the same
        got3 = pt.search(qt, slices=3).view(torch.int64).numpy().view(np.uint64)
        ok_pts = ok_pts and bool(np.array_equal(got3, exp))
        # host buffers in and out (search_host: copies around the routed search)
        oh = torch.empty(q.shape[0], dtype=torch.uint64)
        goth = pt.search_host(qt.clone(), oh).view(torch.int64).numpy().view(np.uint64)
        ok_pts = ok_pts and bool(np.array_equal(goth, exp))
        # ranges: short, long (crossing several shards), empty, lo > hi, full span
        lo1, hi1 = gen.ranges(keys, 200, 40, seed=gen.SEED_RANGE + rank)
        lo2, hi2 = gen.random_ranges(keys, 200, seed=gen.SEED_RANGE + 7 * rank, max_width_keys=T)
        lo = np.concatenate([lo1, lo2, np.array([0, 5, int(keys[-1])], dtype=np.uint64), np.asarray(sp, dtype=np.uint64)])
        hi = np.concatenate([hi1, hi2, np.array([(1 << 64) - 1, 4, (1 << 64) - 1], dtype=np.uint64),
                             np.asarray(sp, dtype=np.uint64) + np.uint64(3)])
        lo, hi = lo.astype(np.uint64), hi.astype(np.uint64)
        tl = torch.from_numpy(lo.view(np.int64).copy()).view(torch.uint64)
        th = torch.from_numpy(hi.view(np.int64).copy()).view(torch.uint64)
        ko, vo, cnt = pt.range(tl, th, cap)
        eko, evo, ecnt = oracle.sorted_range(keys, vals, lo, hi, cap)
        ok_rng = bool(np.array_equal(cnt.numpy(), ecnt.astype(np.int64)))
        if cap:
            k = ko.view(torch.int64).numpy().view(np.uint64)
            v = vo.view(torch.int64).numpy().view(np.uint64)
            m = np.minimum(ecnt.astype(np.int64), cap)
            mask = np.arange(cap)[None, :] < m[:, None]
            ok_rng = ok_rng and bool(np.array_equal(k[mask], eko[mask])) and bool(np.array_equal(v[mask], evo[mask]))
        result_q.put((rank, ok_pts, ok_rng))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,cap", [(1, 16), (2, 16), (3, 0), (3, 64)])
def test_partitioned_exchange_gloo(world, cap):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_worker, args=(r, world, port, 20000, cap, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, ok_pts, ok_rng in res:
        assert ok_pts, f"rank {rank}: point results differ from the oracle"
        assert ok_rng, f"rank {rank}: range results differ from the oracle"


def test_splitters_and_slices():
    from paper_conf_ppopp_yanlpz19_b200.dist import key_splitters

    keys = gen.uniform_keys(1000)
    sp = key_splitters(keys, 4)
    assert sp == [int(keys[250]), int(keys[500]), int(keys[750])]
    assert key_splitters(keys, 1) == []


# ----------------------------------------------------------------------------- peer exchange
class CpuPeerOps:
    """Shared-memory stand-ins for CudaPeerOps (test only): recv[p] / back[p] are CPU tensors in
    shared memory playing the peer-mapped device buffers, the oracle plays the local search."""

    def __init__(self, keys, vals, splitters, P, me, recv, back):
        import oracle

        self.orc, self.keys, self.vals = oracle, keys, vals
        self.split = np.asarray(splitters, dtype=np.uint64)
        self.P, self.me, self.recv, self.back = P, me, recv, back

    def ensure_capacity(self, cap_recv, cap_back):
        assert cap_recv <= self.recv[0].numel() and cap_back <= self.back[0].numel()

    def route_count(self, q):
        self.q = q.view(torch.int64).numpy().view(np.uint64)
        dest = np.searchsorted(self.split, self.q, side="right")
        self.order = np.argsort(dest, kind="stable")  # routed (destination-major) order
        self.dest = dest
        return np.bincount(dest, minlength=self.P).tolist()

    def route_push(self, q, targets):
        qs = self.q[self.order].view(np.int64)
        start = 0
        for d, off in targets:
            c = int(np.sum(self.dest == d))
            self.recv[d][off:off + c] = torch.from_numpy(qs[start:start + c].copy())
            start += c

    def search_recv(self, n):
        qn = self.recv[self.me][:n].numpy().view(np.uint64)
        out = self.orc.sorted_search(self.keys, self.vals, qn, 1)
        return torch.from_numpy(out.view(np.int64).copy())

    def segments_push(self, vals, segs):
        for off, ln, p, doff in segs:
            self.back[p][doff:doff + ln] = vals[off:off + ln]

    def route_return(self, n):
        out = np.empty(n, dtype=np.int64)
        out[self.order] = self.back[self.me][:n].numpy()
        return torch.from_numpy(out).view(torch.uint64)

    def fence(self):
        pass


def _peer_worker(rank, world, port, T, recv, back, result_q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_ppopp_yanlpz19_b200.dist import PeerPartitionedTree, key_splitters

        keys = gen.uniform_keys(T)
        vals = gen.values_for(keys)
        sp = key_splitters(keys, world)
        bounds = [0] + [int(np.searchsorted(keys, np.uint64(s))) for s in sp] + [T]
        lk, lv = keys[bounds[rank]:bounds[rank + 1]], vals[bounds[rank]:bounds[rank + 1]]
        pt = PeerPartitionedTree(lk, lv, sp, ops=CpuPeerOps(lk, lv, sp, world, rank, recv, back))
        ok = True
        for b in range(3):  # several batches through the same buffers, uneven sizes per rank
            nq = 0 if (b == 1 and rank == 0) else 2000 + 300 * rank + 50 * b
            q = np.concatenate([gen.uniform_queries(keys, nq, seed=gen.SEED_QUERY + 10 * b + rank, miss_frac=0.3),
                                np.asarray(sp, dtype=np.uint64)[:nq]])
            got = pt.search(torch.from_numpy(q.view(np.int64).copy()).view(torch.uint64))
            ok = ok and bool(np.array_equal(got.view(torch.int64).numpy().view(np.uint64),
                                            oracle.sorted_search(keys, vals, q)))
        result_q.put((rank, ok))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_peer_exchange_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    recv = [torch.zeros(20000, dtype=torch.int64).share_memory_() for _ in range(world)]
    back = [torch.zeros(20000, dtype=torch.int64).share_memory_() for _ in range(world)]
    procs = [ctx.Process(target=_peer_worker, args=(r, world, port, 20000, recv, back, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, ok in res:
        assert ok, f"rank {rank}: peer-exchange results differ from the oracle"


def test_peer_offsets():
    from paper_conf_ppopp_yanlpz19_b200.dist import peer_offsets

    M = [[1, 2, 3], [4, 5, 6], [7, 8, 9]]  # M[p][d]: queries rank p sends to shard d
    push, roff, rn, boff = peer_offsets(M, 1)
    assert push == [1, 2, 3]          # rank 0's runs precede rank 1's in every receive buffer
    assert roff == [0, 2, 7] and rn == 15  # segments from ranks 0, 1, 2 of shard 1's buffer
    assert boff == [1, 4, 7]          # shard 1's run in each source's routed order


def _update_worker(rank, world, port, T, result_q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_ppopp_yanlpz19_b200.dist import PartitionedTree, key_splitters

        keys = gen.uniform_keys(T)
        vals = gen.values_for(keys)
        sp = key_splitters(keys, world)
        bounds = [0] + [int(np.searchsorted(keys, np.uint64(s))) for s in sp] + [T]
        lk, lv = keys[bounds[rank]:bounds[rank + 1]], vals[bounds[rank]:bounds[rank + 1]]
        pt = PartitionedTree(lk, lv, sp, ops=CpuOps(lk, lv, sp, world))
        ref = oracle.UpdateMap(keys, vals)
        batches = []
        for r in range(world):  # every rank builds every batch (same seeds) for the reference
            n = 0 if r == world - 1 and world > 2 else 3000 + 100 * r
            o, k, v = gen.update_ops(keys, n, insert_frac=0.1, delete_frac=0.2, seed=gen.SEED_OPS + r)
            if n:  # the same key several times inside one batch and across batches
                k[-200:] = k[:200]
                k[:50] = batches[0][1][:50] if batches and len(batches[0][1]) else k[:50]
                o[k == gen.uniform_keys(T)[0]] = 1
            batches.append((o, k, v))
        for o, k, v in batches:
            ref.apply(o, k, v)
        o, k, v = batches[rank]
        t64 = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int64).copy()).view(torch.uint64)
        pt.update(torch.from_numpy(o.copy()), t64(k), t64(v))
        ek, ev = ref.dump()
        q = np.concatenate([keys, np.concatenate([b[1] for b in batches]), gen.edge_queries(keys)])
        got = pt.search(t64(q)).view(torch.int64).numpy().view(np.uint64)
        ok = bool(np.array_equal(got, oracle.sorted_search(ek, ev, q)))
        result_q.put((rank, ok))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [1, 2, 3])
def test_partitioned_update_gloo(world):
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_update_worker, args=(r, world, port, 8000, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, ok in res:
        assert ok, f"rank {rank}: routed updates differ from the global-order oracle"


class CpuTree:
    """Oracle stand-in for one rank's replicated layout (test only)."""

    def __init__(self, keys, vals):
        import oracle

        self.orc, self.keys, self.vals = oracle, keys, vals

    def search(self, q):
        qn = q.view(torch.int64).numpy().view(np.uint64)
        out = self.orc.sorted_search(self.keys, self.vals, qn, 1)
        return torch.from_numpy(out.view(np.int64).copy()).view(torch.uint64)


def _replicated_worker(rank, world, port, T, result_q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_ppopp_yanlpz19_b200.dist import ReplicatedTree

        keys = gen.uniform_keys(T)
        vals = gen.values_for(keys)
        rt = ReplicatedTree(keys, vals, tree=CpuTree(keys, vals))
        q = np.concatenate([gen.uniform_queries(keys, 5001, miss_frac=0.3), gen.edge_queries(keys)])
        qt = torch.from_numpy(q.view(np.int64).copy()).view(torch.uint64)
        b, e = rt.slice_of(q.shape[0])
        mine = rt.search_global(qt).view(torch.int64).numpy().view(np.uint64)
        full = rt.search_global(qt, gather=True).view(torch.int64).numpy().view(np.uint64)
        exp = oracle.sorted_search(keys, vals, q)
        result_q.put((rank, bool(np.array_equal(mine, exp[b:e])), bool(np.array_equal(full, exp)), e - b))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_replicated_gloo(world):
    """Replicated mode: rank p answers [p*Q/P, (p+1)*Q/P) with no collective;
    the slices tile the batch and the gathered result equals the oracle."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_replicated_worker, args=(r, world, port, 6000, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    assert sum(r[3] for r in res) == 5001 + len(gen.edge_queries(gen.uniform_keys(6000)))
    for rank, ok_slice, ok_full, _ in res:
        assert ok_slice and ok_full, rank


def _reject_worker(rank, world, port, T, result_q):
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        import oracle
        from paper_conf_ppopp_yanlpz19_b200 import HarmoniaError
        from paper_conf_ppopp_yanlpz19_b200.dist import PartitionedTree, key_splitters

        keys = gen.uniform_keys(T)
        vals = gen.values_for(keys)
        sp = key_splitters(keys, world)
        bounds = [0] + [int(np.searchsorted(keys, np.uint64(s))) for s in sp] + [T]
        lk, lv = keys[bounds[rank]:bounds[rank + 1]], vals[bounds[rank]:bounds[rank + 1]]
        pt = PartitionedTree(lk, lv, sp, ops=CpuOps(lk, lv, sp, world))
        o, k, v = gen.update_ops(keys, 500, insert_frac=0.1, seed=gen.SEED_OPS + rank)
        if rank == 1:
            k[7] = np.uint64(0xFFFFFFFFFFFFFFFF)  # a reserved key in one rank's batch only
        t64 = lambda a: torch.from_numpy(np.ascontiguousarray(a).view(np.int64).copy()).view(torch.uint64)
        status = None
        try:
            pt.update(torch.from_numpy(o.copy()), t64(k), t64(v))
        except HarmoniaError as e:
            status = e.status
        got = pt.search(t64(keys)).view(torch.int64).numpy().view(np.uint64)
        result_q.put((rank, status, bool(np.array_equal(got, oracle.sorted_search(keys, vals, keys)))))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world", [2, 3])
def test_partitioned_update_rejects_everywhere(world):
    """A reserved key in ONE rank's batch: every rank raises HARMONIA_ERR_RESERVED before any
    shard applies an op, and every shard is unchanged."""
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_reject_worker, args=(r, world, port, 6000, q)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=240) for _ in range(world)]
    for p in procs:
        p.join(timeout=60)
        assert p.exitcode == 0
    for rank, status, unchanged in res:
        assert status == 3 and unchanged, (rank, status, unchanged)
