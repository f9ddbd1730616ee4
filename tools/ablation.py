"""Design-choice ablation on B200 (the paper's Figs 8 and 13) and the NTG
model against the measured group-size sweep (f4).

  python tools/ablation.py --what ablation  > profiles/rNN_ablation.jsonl
  python tools/ablation.py --what ntg_model > profiles/rNN_ntg_model.jsonl

ablation (log2 T = 23..26, F = 64, Q = 2^26 uniform hits; one JSON line per variant):
  tree_only       Harmonia layout, G = F/2 (one 128-bit step per node), PSA off
  psa             + PSA (Eq 2 bits, two-level partition), G = F/2
  psa_ntg_model   + NTG with the paper's linear walk at the Eq 3/4 model's G
  psa_ntg_kary    + NTG, k-ary in-node steps at G = 2 (the best ballot group measured)
  default         the library default (PSA + G = 1 warp-shared descent, staged return)
  full_sort       comparator: a full radix sort of the batch (torch.sort = CUB) + search of
                  the sorted batch (PSA off) + scatter back (P:L336 calls this a net loss)
  Also the PSA kernels alone (library profile) against the full sort alone.
ntg_model (T = 2^26, F = 8..128, fill 1.0 and 0.69, Zipf theta 0.99 queries as config 3):
  the Eq 3/4 choice from 1000 samples (harmonia_tune_group_size) against the measured
  throughput of every G with the paper's linear NTG walk and with the k-ary walk.
CUDA-event timing on the launch stream after warm-up; inputs resident in HBM.
"""
import argparse
import json
import os
import sys

import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import harmonia_gen as gen  # noqa: E402
import paper_conf_ppopp_yanlpz19_b200 as hm  # noqa: E402


def timed(fn, reps):
    s0, s1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
    for _ in range(2):
        fn()
    torch.cuda.synchronize()
    s0.record()
    for _ in range(reps):
        fn()
    s1.record()
    torch.cuda.synchronize()
    return s0.elapsed_time(s1) / reps


def emit(d):
    print(json.dumps(d), flush=True)


SIGN = -(1 << 63)


def ablation(reps, Q=1 << 26, F=64):
    for lt in (23, 24, 25, 26):
        T = 1 << lt
        keys = gen.uniform_keys_t(T, "cuda")
        vals = gen.values_for_t(keys)
        t = hm.Tree(keys, vals, fanout=F)
        q = gen.uniform_queries_t(keys, Q)
        out = torch.empty_like(q)
        gm, steps = t.tune_group_size(q[:1000])
        expect = gen.values_for_t(q)  # every query is a hit: the result is its key's value
        variants = [("tree_only", dict(group_size=F // 2, psa_bits=-1)),
                    ("psa", dict(group_size=F // 2)),
                    ("psa_ntg_model", dict(group_size=gm, flags=hm.QF_LINEAR)),
                    ("psa_ntg_kary", dict(group_size=2)),
                    ("default", dict())]
        for name, kw in variants:
            o = hm.make_opts(**kw)
            ms = timed(lambda: t.search(q, out, opts=o), reps)
            ok = bool(torch.equal(out, expect))
            hm.profile_enable(True)
            hm.profile_read()
            t.search(q, out, opts=o)
            pr = hm.profile_read()
            hm.profile_enable(False)
            emit({"what": "ablation", "T": T, "F": F, "Q": Q, "variant": name, "opts": kw, "ms": ms,
                  "Gq_per_s": Q / ms / 1e6, "parity": ok, "model_G": gm,
                  "kernels_ms": {k: v[0] for k, v in pr.items()}})
        # full sort comparator (CUB radix sort through torch) + search sorted + scatter back
        o = hm.make_opts(group_size=1, psa_bits=-1)
        qi = q.view(torch.int64)

        def full_sort_path():
            s, idx = torch.sort(qi ^ SIGN)  # unsigned order via the flipped sign bit
            res = t.search((s ^ SIGN).view(torch.uint64), opts=o)
            out.view(torch.int64).index_copy_(0, idx, res.view(torch.int64))

        ms = timed(full_sort_path, reps)
        ok = bool(torch.equal(out, expect))
        ms_sort = timed(lambda: torch.sort(qi ^ SIGN), reps)
        hm.profile_enable(True)
        hm.profile_read()
        t.search(q, out)
        pr = hm.profile_read()
        hm.profile_enable(False)
        psa_ms = sum(pr[k][0] for k in ("psa_hist", "psa_scan", "psa_scatter") if k in pr)
        emit({"what": "ablation", "T": T, "F": F, "Q": Q, "variant": "full_sort", "ms": ms, "Gq_per_s": Q / ms / 1e6,
              "parity": ok, "sort_only_ms": ms_sort, "psa_only_ms": psa_ms,
              "psa_over_full_sort": psa_ms / ms_sort})
        t.close()
        del keys, vals, q, out, expect
        torch.cuda.empty_cache()


def ntg_model(reps, T=1 << 26, Q=1 << 26):
    keys = gen.uniform_keys_t(T, "cuda")
    vals = gen.values_for_t(keys)
    q = torch.from_numpy(gen.zipf_queries(keys.cpu().numpy(), Q)).cuda()
    out = torch.empty_like(q)
    for F in (8, 16, 32, 64, 128):
        for fill in (1.0, 0.69):
            t = hm.Tree(keys, vals, fanout=F, fill=fill)
            gm, steps = t.tune_group_size(q[:1000])
            rows = {}
            for mode, flags in (("linear", hm.QF_LINEAR), ("kary", 0)):
                for G in (2, 4, 8, 16, 32):
                    if 2 * G > F:
                        continue
                    o = hm.make_opts(group_size=G, flags=flags)
                    ms = timed(lambda: t.search(q, out, opts=o), reps)
                    rows[(mode, G)] = Q / ms / 1e6
            lin = {G: v for (m, G), v in rows.items() if m == "linear"}
            best = max(lin, key=lin.get)
            emit({"what": "ntg_model_vs_sweep", "T": T, "F": F, "fill": fill, "Q": Q, "dist": "zipf0.99",
                  "height": t.info()["height"], "model_G": gm, "model_S": steps,
                  "linear_Gq_per_s": lin, "kary_Gq_per_s": {G: v for (m, G), v in rows.items() if m == "kary"},
                  "best_linear_G": best, "model_over_best_linear": lin[gm] / lin[best],
                  "default_G1_Gq_per_s": Q / timed(lambda: t.search(q, out), reps) / 1e6})
            t.close()
            torch.cuda.empty_cache()


if __name__ == "__main__":
    ap = argparse.ArgumentParser()
    ap.add_argument("--what", default="ablation,ntg_model")
    ap.add_argument("--reps", type=int, default=5)
    a = ap.parse_args()
    for w in a.what.split(","):
        {"ablation": ablation, "ntg_model": ntg_model}[w](a.reps)
