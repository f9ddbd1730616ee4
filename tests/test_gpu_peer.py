"""Fused routing over peer memory (harmonia_route_count / route_push / segments_push /
route_return, CUDA IPC buffers) on the GPU, bit-exact against the oracle.

* single process: P virtual shards whose receive and back buffers are slices of local
  tensors, so every kernel of the exchange runs without IPC;
* two processes on the same GPU (gloo for the small control collectives): the full
  PeerPartitionedTree path with real CUDA IPC mappings of the peer buffers (the box has one
  GPU; across GPUs the same stores go over NVLink)."""
import os
import socket

import numpy as np
import pytest
import torch

import harmonia_gen as gen

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def hm():
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    import paper_conf_ppopp_yanlpz19_b200 as m

    m.lib()
    return m


def _u64(a):
    return torch.from_numpy(np.ascontiguousarray(a, dtype=np.uint64).view(np.int64)).view(torch.uint64).cuda()


def _np(t):
    return t.view(torch.int64).cpu().numpy().view(np.uint64)


@pytest.mark.parametrize("P,n", [(1, 1000), (3, 50001), (7, 4096), (64, 100000), (256, 30000)])
def test_route_push_return_single_process(hm, orc, P, n):
    keys = gen.uniform_keys(1 << 16)
    vals = gen.values_for(keys)
    sp = [int(keys[(p * len(keys)) // P]) for p in range(1, P)]
    q = np.concatenate([gen.uniform_queries(keys, n, miss_frac=0.2), np.asarray(sp, dtype=np.uint64)])
    qd = _u64(q)
    spd = _u64(np.asarray(sp if sp else [0], dtype=np.uint64))
    ws = hm.route_workspace(P, qd.numel(), qd.device)
    counts = hm.route_count(spd, P, qd, ws)
    dest = np.searchsorted(np.asarray(sp, dtype=np.uint64), q, side="right")
    assert counts == np.bincount(dest, minlength=P).tolist()
    # every shard's receive buffer is a slice of `recv`, with a gap so stray writes show up
    gap = 5
    starts = np.concatenate([[0], np.cumsum(np.asarray(counts) + gap)])[:P]
    recv = torch.full((int(starts[-1]) + counts[-1] + gap,), -7, dtype=torch.int64, device="cuda")
    hm.route_push(spd, P, qd, [recv.data_ptr() + 8 * int(s) for s in starts], ws)
    torch.cuda.synchronize()
    r = recv.cpu().numpy().view(np.uint64)
    for d in range(P):
        run = r[starts[d]:starts[d] + counts[d]]
        assert np.array_equal(np.sort(run), np.sort(q[dest == d]))  # order inside a run: unspecified
        assert np.all(recv.cpu().numpy()[starts[d] + counts[d]:starts[d] + counts[d] + gap] == -7)
    # answer each run, push the answers back into one routed-order buffer, invert the partition
    res = torch.from_numpy(orc.sorted_search(keys, vals, r).view(np.int64)).cuda()
    back = torch.full((qd.numel(),), -1, dtype=torch.int64, device="cuda")
    excl = np.concatenate([[0], np.cumsum(counts)])[:P]
    ws2 = hm.route_workspace(1, 1, qd.device)
    hm.segments_push(res, [int(s) for s in starts], counts, [back.data_ptr() + 8 * int(e) for e in excl], ws2)
    out = torch.empty_like(qd)
    hm.route_return(P, back.data_ptr(), qd.numel(), out, ws)
    assert np.array_equal(_np(out), orc.sorted_search(keys, vals, q))


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _ipc_worker(rank, world, port, T, result_q, device_barrier=True):
    import torch.distributed as dist

    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    dist.init_process_group("gloo", rank=rank, world_size=world)
    try:
        torch.cuda.set_device(0)
        import oracle
        from paper_conf_ppopp_yanlpz19_b200.dist import PeerPartitionedTree, key_splitters

        keys = gen.uniform_keys(T)
        vals = gen.values_for(keys)
        sp = key_splitters(keys, world)
        bnd = [0] + [int(np.searchsorted(keys, np.uint64(s))) for s in sp] + [T]
        lk, lv = keys[bnd[rank]:bnd[rank + 1]], vals[bnd[rank]:bnd[rank + 1]]
        pt = PeerPartitionedTree(_u64(lk), _u64(lv), sp, fanout=16, device=torch.device("cuda", 0),
                                 device_barrier=device_barrier)
        ok = True
        for b, nq in enumerate((3000, 0, 70000, 5000)):  # growth of the buffers, an empty batch
            nq = nq + 111 * rank if nq else (0 if rank == 0 else 900)
            q = np.concatenate([gen.uniform_queries(keys, nq, seed=gen.SEED_QUERY + 10 * b + rank, miss_frac=0.3),
                                gen.edge_queries(keys) if nq else np.zeros(0, np.uint64)])
            got = _np(pt.search(_u64(q)))
            ok = ok and bool(np.array_equal(got, oracle.sorted_search(keys, vals, q)))
        pt.close()
        result_q.put((rank, ok, ""))
    except Exception as e:  # report instead of hanging the parent
        result_q.put((rank, False, repr(e)))
    finally:
        dist.destroy_process_group()


@pytest.mark.parametrize("world,device_barrier", [(2, True), (3, True), (2, False)])
def test_peer_partitioned_two_processes_ipc(world, device_barrier):
    """device_barrier: the batch's two barriers are harmonia_peer_barrier kernels (flags in
    IPC-mapped peer memory); False: stream synchronise + host barrier."""
    import torch.multiprocessing as mp

    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    procs = [ctx.Process(target=_ipc_worker, args=(r, world, port, 60000, q, device_barrier)) for r in range(world)]
    for p in procs:
        p.start()
    res = [q.get(timeout=300) for _ in range(world)]
    for p in procs:
        p.join(timeout=120)
    for rank, ok, err in res:
        assert ok, f"rank {rank}: {err or 'peer-routed results differ from the oracle'}"


@pytest.mark.parametrize("P", [1, 3, 8])
def test_peer_barrier_single_process(hm, P):
    """harmonia_peer_barrier with P virtual ranks in one process, each on its own stream: every
    kernel returns only when all P have arrived, with every flag at the epoch; a rank whose
    peers never arrive times out and reports it instead of hanging."""
    bufs = [torch.zeros(P, dtype=torch.int64, device="cuda") for _ in range(P)]  # rank me's flag array
    addrs = torch.tensor([b.data_ptr() for b in bufs], dtype=torch.int64, device="cuda")
    err = torch.zeros(1, dtype=torch.int32, device="cuda")
    streams = [torch.cuda.Stream() for _ in range(P)]
    for epoch in (1, 2, 3):
        for me in range(P):
            hm.peer_barrier(P, me, addrs, bufs[me].data_ptr(), epoch, err, stream=streams[me])
        torch.cuda.synchronize()
        assert int(err.item()) == 0
        for b in bufs:
            assert b.cpu().tolist() == [epoch] * P
    if P > 1:  # only rank 0 arrives at epoch 4: it must time out (1 ms), not hang
        hm.peer_barrier(P, 0, addrs, bufs[0].data_ptr(), 4, err, timeout_ns=1_000_000)
        torch.cuda.synchronize()
        assert int(err.item()) == 1


@pytest.mark.parametrize("P,cap", [(1, 16), (3, 0), (4, 64), (16, 32)])
def test_range_split_assemble_single_process(hm, orc, P, cap):
    """harmonia_range_split_count/_emit cut ranges at the splitters, P shard trees answer their
    pieces (harmonia_range_batch), harmonia_range_assemble reassembles: equal to the oracle on
    the whole key set (slab contents up to min(count, cap) and true totals)."""
    T = 40000
    keys = gen.uniform_keys(T)
    vals = gen.values_for(keys)
    sp = [int(keys[(p * T) // P]) for p in range(1, P)]
    bnd = [0] + [int(np.searchsorted(keys, np.uint64(s))) for s in sp] + [T]
    trees = [hm.Tree(_u64(keys[bnd[d]:bnd[d + 1]]), _u64(vals[bnd[d]:bnd[d + 1]]), fanout=16) for d in range(P)]
    lo1, hi1 = gen.ranges(keys, 3000, 40)
    lo2, hi2 = gen.random_ranges(keys, 3000, max_width_keys=T)
    spa = np.asarray(sp, dtype=np.uint64)
    lo = np.concatenate([lo1, lo2, np.array([0, 5, int(keys[-1])], dtype=np.uint64), spa, spa - np.uint64(1)]).astype(np.uint64)
    hi = np.concatenate([hi1, hi2, np.array([(1 << 64) - 1, 4, (1 << 64) - 1], dtype=np.uint64), spa + np.uint64(3), spa]).astype(np.uint64)
    spd = _u64(spa if P > 1 else np.zeros(1, np.uint64))
    plo, phi, pid, counts, pbase = hm.range_split(spd, P, _u64(lo), _u64(hi))
    m = plo.numel()
    assert sum(counts) == m
    rc = torch.empty(m, dtype=torch.int32, device="cuda")
    rk = torch.empty(max(m * cap, 1), dtype=torch.uint64, device="cuda")
    rv = torch.empty(max(m * cap, 1), dtype=torch.uint64, device="cuda")
    start = 0
    for d in range(P):  # each destination run answered by its shard
        c = counts[d]
        if c:
            ko, vo, cnt = trees[d].range(plo[start:start + c], phi[start:start + c], cap)
            rc[start:start + c] = cnt.view(torch.int32)
            if cap:
                rk[start * cap:(start + c) * cap] = ko.reshape(-1)
                rv[start * cap:(start + c) * cap] = vo.reshape(-1)
        start += c
    ko, vo, tot = hm.range_assemble(len(lo), cap, pbase, pid, rc, rk, rv)
    eko, evo, ecnt = orc.sorted_range(keys, vals, lo, hi, cap)
    assert np.array_equal(_np(tot), ecnt.astype(np.uint64))
    if cap:
        mk = np.arange(cap)[None, :] < np.minimum(ecnt.astype(np.int64), cap)[:, None]
        gk, gv = _np(ko).reshape(-1, cap), _np(vo).reshape(-1, cap)
        assert np.array_equal(gk[mk], eko.reshape(-1, cap)[mk]) and np.array_equal(gv[mk], evo.reshape(-1, cap)[mk])
        assert np.all(gk[~mk] == np.uint64((1 << 64) - 1))


def test_partitioned_single_rank_with_updates(hm, orc):
    """Config 5's loop at N = 1 on the GPU: a one-rank NCCL group, PartitionedTree (routing
    bypassed at P = 1) over a fill-0.69 shard, query batches interleaved with 5 % insert / 5 %
    delete / 90 % update batches (in place), every batch checked against the std::map oracle."""
    import torch.distributed as dist

    from paper_conf_ppopp_yanlpz19_b200.dist import PartitionedTree

    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    port = s.getsockname()[1]
    s.close()
    dist.init_process_group("nccl", init_method=f"tcp://127.0.0.1:{port}", rank=0, world_size=1,
                            device_id=torch.device("cuda", 0))
    try:
        keys = gen.uniform_keys(1 << 18)
        vals = gen.values_for(keys)
        pt = PartitionedTree(_u64(keys), _u64(vals), [], fanout=64, fill=0.69, device=torch.device("cuda", 0))
        ref = orc.UpdateMap(keys, vals)
        modes = []
        for b in range(4):
            rk, rv = ref.dump()
            q = gen.uniform_queries(rk, 300000, seed=gen.SEED_QUERY + b, miss_frac=0.2)
            assert np.array_equal(_np(pt.search(_u64(q))), orc.sorted_search(rk, rv, q))
            ops, ks, vs = gen.update_ops(rk, 20000, insert_frac=0.05, delete_frac=0.05, seed=gen.SEED_OPS + b)
            pt.update(torch.from_numpy(ops).cuda(), _u64(ks), _u64(vs))
            modes.append(pt.ops.tree.last_update_mode())
            ref.apply(ops, ks, vs)
        rk, rv = ref.dump()
        q = np.concatenate([rk, gen.edge_queries(rk)])
        assert np.array_equal(_np(pt.search(_u64(q))), orc.sorted_search(rk, rv, q))
        assert modes.count(1) >= 3, modes
    finally:
        dist.destroy_process_group()
