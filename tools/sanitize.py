"""Measurement helper (not product code): a small driver that launches every kernel family of
libharmonia.so once or twice on small inputs, for compute-sanitizer runs
(memcheck / racecheck / synccheck / initcheck; tools/gpu_sanitize.sh).  Results are checked
against the generator's closed form (value = values_for(key) for a hit, NOT_FOUND for a miss)
so a run that corrupts memory also fails here.

    PYTORCH_NO_CUDA_MEMORY_CACHING=1 compute-sanitizer --tool memcheck python tools/sanitize.py
"""
import os
import sys

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import harmonia_gen as gen  # noqa: E402
import paper_conf_ppopp_yanlpz19_b200 as hm  # noqa: E402

SMALL = os.environ.get("SANITIZE_SMALL", "0") == "1"


def cu(a):
    return torch.from_numpy(np.ascontiguousarray(a)).cuda()


def expect(keys, q):
    hit = np.isin(q, keys)
    return np.where(hit, gen.values_for(q), np.uint64(hm.NOT_FOUND)).astype(np.uint64)


def check(name, got, want):
    got = got.cpu().numpy() if hasattr(got, "cpu") else got
    ok = np.array_equal(got, want)
    print(f"{name}: {'ok' if ok else 'MISMATCH'}", flush=True)
    if not ok:
        sys.exit(1)


def main():
    n_keys = 3000 if SMALL else 40_000
    n_q = 20_000 if SMALL else 150_001
    for F, fill in ((8, 0.69), (64, 1.0), (128, 0.5)):
        keys = gen.uniform_keys(n_keys)
        vals = gen.values_for(keys)
        t = hm.Tree(cu(keys), cu(vals), fanout=F, fill=fill)
        q = np.concatenate([gen.uniform_queries(keys, n_q, miss_frac=0.3), gen.edge_queries(keys)])
        want = expect(keys, q)
        qd = cu(q)
        check(f"F{F} default", t.search(qd), want)
        for name, kw in (("L16", dict(flags=hm.QF_PSA_L16, psa_bits=16)), ("L8", dict(flags=hm.QF_PSA_L8)),
                         ("global", dict(flags=hm.QF_PSA_GLOBAL)), ("scatter", dict(flags=hm.QF_SCATTER_RETURN)),
                         ("gather", dict(flags=hm.QF_GATHER)), ("per_lane", dict(flags=hm.QF_PER_LANE)),
                         ("G4", dict(group_size=4)), ("G4 linear", dict(group_size=4, flags=hm.QF_LINEAR)),
                         ("no psa", dict(psa_bits=-1)), ("no smem", dict(flags=hm.QF_NO_PS_SMEM))):
            check(f"F{F} {name}", t.search(qd, **kw), want)
        check(f"F{F} tiny batch", t.search(cu(q[:37])), want[:37])
        out_h = t.search_host(q[:5000])
        torch.cuda.synchronize()  # asynchronous on the stream, like the C call
        check(f"F{F} host", out_h, want[:5000])
        # ranges: lane kernel (cap < 512), warp kernel (cap >= 512), G-group walk
        lo, hi = gen.ranges(keys, 2000, 16)
        lod, hid = cu(lo), cu(hi)
        for cap, kw in ((16, {}), (600, {}), (16, dict(flags=hm.QF_RANGE_GROUP))):
            rk, rv, cnt = t.range(lod, hid, cap, **kw)
            s = np.searchsorted(keys, lo)
            e = np.searchsorted(keys, hi, side="right")
            check(f"F{F} range cap{cap} {kw}", cnt.cpu().numpy().astype(np.int64), (e - s).astype(np.int64))
            rk = rk.cpu().numpy()
            first = np.array([keys[s[i]] for i in range(len(lo))], dtype=np.uint64)
            check(f"F{F} range cap{cap} first key", rk[:, 0], first)
        # update batches: in place (fill < 1) and the rebuild (fill 1.0)
        ops, uk, uv = gen.update_ops(keys, 4096, insert_frac=0.05, delete_frac=0.05)
        t.update(cu(ops), cu(uk), cu(uv))
        torch.cuda.synchronize()
        print(f"F{F} update mode {t.last_update_mode()}", flush=True)
        t.search(qd)
        g = t.tune_group_size(qd[:4096])
        print(f"F{F} tune G={g}", flush=True)
        t.close()
    # multi-GPU routing kernels (one process: P virtual shards)
    keys = gen.uniform_keys(n_keys)
    q = cu(gen.uniform_queries(keys, n_q))
    spl = cu(keys[[n_keys // 4, n_keys // 2, 3 * n_keys // 4]])
    res = hm.route_partition(spl, 4, q)
    torch.cuda.synchronize()
    print("route ok", flush=True)
    del res
    torch.cuda.synchronize()
    print("SANITIZE DONE", flush=True)


if __name__ == "__main__":
    main()
