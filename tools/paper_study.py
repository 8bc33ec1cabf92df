"""NEXT-3 study on B200: the paper's comparison shape on the
synthetic C1-C5 workloads, three arms timed on the same data and device:

  * sweet  -- the default join (this library's Sweet KNN path);
  * basic  -- mapping='basic': the basic KNN-TI Sweet KNN starts from
              (Fig. 4 / Alg. 2, thread per query in input order, no remap;
              P:L733-767 "KNN-TI" columns of Fig. 9 / Table IV);
  * gemm   -- a library brute force standing in for the paper's cuBLAS-based
              KNN baseline: ||q||^2 + ||t||^2 - 2 Q T^T with
              torch.matmul (cuBLAS, fp32) in query chunks + torch.topk. Not
              exact (the expansion rounds differently), context only.

    python tools/paper_study.py [--configs C1,C2,C3,C4,C5] [--reps 5]
                                [--gemm-sample 16384] [--arms sweet,basic,gemm]

One JSON line per (config, arm): ms per join (median of reps, CUDA events on
the launching stream after a warm-up), queries/s, % pruned, distance
evaluations. For C4/C5 the basic and gemm arms run on a seeded query sample
against all targets (their cost per query is independent of the other
queries for gemm; for basic the sample's clusters are re-built, so its line
says `sample`), and queries/s is reported for the sample. Warp efficiency
(Table IV's metric) comes from ncu, tools/paper_study_ncu.sh.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import datagen  # noqa: E402


def time_ms(fn, reps):
    import torch
    fn()
    torch.cuda.synchronize()
    s = torch.cuda.current_stream()
    out = []
    for _ in range(reps):
        a = torch.cuda.Event(enable_timing=True)
        b = torch.cuda.Event(enable_timing=True)
        a.record(s)
        fn()
        b.record(s)
        torch.cuda.synchronize()
        out.append(a.elapsed_time(b))
    out.sort()
    return out[len(out) // 2]


def gemm_knn(dQ, dT, k, budget_bytes=4 << 30):
    """Brute force through cuBLAS: distance matrix per query chunk, then topk."""
    import torch
    tn = (dT * dT).sum(1)
    nt = dT.shape[0]
    b = max(1, min(dQ.shape[0], budget_bytes // (4 * nt)))
    outs_i, outs_d = [], []
    for s0 in range(0, dQ.shape[0], b):
        q = dQ[s0:s0 + b]
        D = torch.addmm(tn[None, :], q, dT.t(), beta=1.0, alpha=-2.0)
        D += (q * q).sum(1, keepdim=True)
        d, i = torch.topk(D, k, dim=1, largest=False, sorted=True)
        outs_i.append(i)
        outs_d.append(d.clamp_min_(0).sqrt_())
    return torch.cat(outs_i), torch.cat(outs_d)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C1,C2,C3,C4,C5")
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--arms", default="sweet,basic,gemm")
    ap.add_argument("--gemm-sample", type=int, default=16384)
    ap.add_argument("--basic-sample", type=int, default=65536)
    args = ap.parse_args()
    import torch
    import paper_conf_icde_chends17_b200 as sknn
    torch.backends.cuda.matmul.allow_tf32 = False
    arms = args.arms.split(",")
    for name in args.configs.split(","):
        Q, T, k, sj = datagen.workload(name)
        dQ = torch.from_numpy(Q).cuda()
        dT = dQ if sj else torch.from_numpy(T).cuda()
        for arm in arms:
            rec = {"config": name, "arm": arm, "nq": int(Q.shape[0]), "nt": int(T.shape[0]), "d": int(Q.shape[1]),
                   "k": int(k)}
            if arm == "sweet":
                ms = time_ms(lambda: sknn.join(dQ, dT, k), args.reps)
                _, _, st = sknn.join(dQ, dT, k, stats=True)
                rec.update(ms=ms, nq_timed=int(Q.shape[0]), pruned_pct=st["pruned_pct"],
                           evals=int(st["dist_evals_sparse"] + st["dist_evals_dense"]))
            elif arm == "basic":
                qs = dQ
                tgt = dT
                if Q.shape[0] > args.basic_sample:  # seeded sample of queries, all targets
                    rng = np.random.default_rng(99)
                    s = np.sort(rng.choice(Q.shape[0], args.basic_sample, replace=False))
                    qs = torch.from_numpy(Q[s]).cuda()
                    rec["sample"] = "%d seeded queries (seed 99) x all targets, Q != T join" % len(s)
                    # the Sweet arm on the same sample, for a like-for-like ratio
                    rec["ms_sweet_same_sample"] = time_ms(lambda: sknn.join(qs, tgt, k), args.reps)
                ms = time_ms(lambda: sknn.join(qs, tgt, k, mapping="basic"), max(1, args.reps // 2))
                _, _, st = sknn.join(qs, tgt, k, stats=True, mapping="basic")
                rec.update(ms=ms, nq_timed=int(qs.shape[0]), pruned_pct=st["pruned_pct"],
                           evals=int(st["dist_evals_sparse"]))
            elif arm == "gemm":
                qs = dQ
                if Q.shape[0] > args.gemm_sample:
                    rng = np.random.default_rng(99)
                    s = np.sort(rng.choice(Q.shape[0], args.gemm_sample, replace=False))
                    qs = torch.from_numpy(Q[s]).cuda()
                    rec["sample"] = "%d seeded queries (seed 99) x all targets" % len(s)
                ms = time_ms(lambda: gemm_knn(qs, dT, k), max(1, args.reps // 2))
                rec.update(ms=ms, nq_timed=int(qs.shape[0]), pruned_pct=0.0,
                           evals=int(qs.shape[0]) * int(T.shape[0]))
            rec["queries_per_s"] = rec["nq_timed"] / (rec["ms"] / 1e3)
            print(json.dumps(rec), flush=True)
        del dQ, dT
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
