"""Sharded clustering (NEXT-1), one rank's share measured on one GPU: the
full build (sknn_build) vs rank 0's sknn_build_assign_shard at P = 2/4/8 plus
sknn_build_from_assignment (each rank runs both; the all-reduce of 8 bytes
per point is not included). CUDA events, median of reps.

    python tools/sharded_build_bench.py [--config C5] [--side Q] [--reps 3]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))

import datagen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C5")
    ap.add_argument("--side", default="Q")
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    import torch
    import paper_conf_icde_chends17_b200 as sknn
    from paper_conf_icde_chends17_b200.dist import aligned_bounds
    from tools_timing import time_ms
    Q, T, k, sj = datagen.workload(args.config)
    X = torch.from_numpy(Q if args.side == "Q" else T).cuda()
    full = time_ms(lambda: sknn.build(X).close(), args.reps)
    print(json.dumps({"config": args.config, "side": args.side, "n": int(X.shape[0]), "P": 1, "ms": full}), flush=True)
    for P in (2, 4, 8):
        lo, hi = aligned_bounds(X.shape[0], P, 0)
        ms_a = time_ms(lambda: sknn.build_assign_shard(X, lo, hi), args.reps)
        c, i, d = sknn.build_assign_shard(X, 0, X.shape[0])
        ms_f = time_ms(lambda: sknn.Index.from_assignment(X, c, i, d).close(), args.reps)
        print(json.dumps({"config": args.config, "side": args.side, "n": int(X.shape[0]), "P": P,
                          "ms_assign_shard": ms_a, "ms_from_assignment": ms_f, "ms": ms_a + ms_f,
                          "vs_full": (ms_a + ms_f) / full}), flush=True)


if __name__ == "__main__":
    main()
