"""Query-sharding load balance, measured on ONE GPU: every
rank's share of a query-sharded join is run on its own (what rank r's GPU
would run: the replicated build + level-1, then its query clusters' scan),
for the interleaved (c % P) and the balanced (shard_policy = 1, snake deal by
the level-1 work estimate) ownership. Reports per policy and P the max and
mean over ranks of the per-rank join time and of the level-2 scan + dense
stage time (CUDA events / sknn_stats), i.e. the step time a P-GPU run would
see (max over ranks) and its imbalance (max / mean).

    python tools/shard_balance.py [--config C4] [--P 2,4,8] [--reps 3]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import datagen  # noqa: E402
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C4")
    ap.add_argument("--P", default="2,4,8")
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    import torch
    import paper_conf_icde_chends17_b200 as sknn
    from tools_timing import time_ms
    Q, T, k, sj = datagen.workload(args.config)
    dQ = torch.from_numpy(Q).cuda()
    dT = dQ if sj else torch.from_numpy(T).cuda()
    full = time_ms(lambda: sknn.join(dQ, dT, k), args.reps)
    print(json.dumps({"config": args.config, "P": 1, "ms": full}), flush=True)
    for P in [int(x) for x in args.P.split(",")]:
        for pol in (0, 1):
            per, stage = [], []
            for r in range(P):
                o = dict(shard_rank=r, shard_count=P, shard_policy=pol)
                per.append(time_ms(lambda: sknn.join(dQ, dT, k, **o), args.reps))
                _, _, st = sknn.join(dQ, dT, k, stats=True, **o)
                stage.append(st["ms_sparse"] + st["ms_dense"])
            emit(args.config, P, ["interleave", "balanced"][pol], per, stage)
        if not sj:  # dist.py's Q != T mode: contiguous query row slices, each clustered on its own rank
            per, stage = [], []
            for r in range(P):
                lo, hi = r * Q.shape[0] // P, (r + 1) * Q.shape[0] // P
                qr = dQ[lo:hi].contiguous()
                per.append(time_ms(lambda: sknn.join(qr, dT, k), args.reps))
                _, _, st = sknn.join(qr, dT, k, stats=True)
                stage.append(st["ms_sparse"] + st["ms_dense"])
            emit(args.config, P, "row-slices", per, stage)


def emit(config, P, policy, per, stage):
    print(json.dumps({"config": config, "P": P, "policy": policy,
                      "ms_max": max(per), "ms_mean": sum(per) / P, "imbalance": max(per) / (sum(per) / P),
                      "scan_ms_max": max(stage), "scan_ms_mean": sum(stage) / P,
                      "scan_imbalance": max(stage) / (sum(stage) / P), "per_rank_ms": per}), flush=True)


if __name__ == "__main__":
    main()
