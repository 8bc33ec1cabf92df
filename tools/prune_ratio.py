"""NEXT-1 exchange pruning, measured on one GPU: the partial k-lists of P
target shards (each shard's join run in turn, as rank r would), then the
fraction of entries at or below the per-query minimum over shards of the
local k-th squared distance -- the entries a pruned all-to-all still moves --
and a check that merging only those gives the unpruned merge's result.

    python tools/prune_ratio.py [--config C5] [--P 2,4,8] [--nq 500000]
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import datagen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C5")
    ap.add_argument("--P", default="2,4,8")
    ap.add_argument("--nq", type=int, default=500_000, help="queries used (a prefix; all targets)")
    args = ap.parse_args()
    import torch
    import paper_conf_icde_chends17_b200 as sknn
    from paper_conf_icde_chends17_b200.dist import shard_bounds
    Q, T, k, sj = datagen.workload(args.config)
    Q = Q[:args.nq]
    dQ = torch.from_numpy(Q).cuda()
    dT = torch.from_numpy(T).cuda()
    for P in [int(x) for x in args.P.split(",")]:
        pi, pd = [], []
        for r in range(P):
            lo, hi = shard_bounds(T.shape[0], P, r)
            i, d = sknn.join(dQ, dT[lo:hi].contiguous(), k, out_squared=1, index_base=lo)
            pi.append(i)
            pd.append(d)
        PI, PD = torch.stack(pi), torch.stack(pd)
        kth = PD[:, :, k - 1].min(0).values
        keep = PD <= kth[None, :, None]
        frac = keep.float().mean().item()
        full_i, full_d = sknn.merge_partials(PI, PD, k, out_squared=True)
        pruned_d = torch.where(keep, PD, torch.full_like(PD, float("inf")))
        pruned_i = torch.where(keep, PI, torch.full_like(PI, -1))
        pr_i, pr_d = sknn.merge_partials(pruned_i, pruned_d, k, out_squared=True)
        same = bool(torch.equal(full_i, pr_i) and torch.equal(full_d, pr_d))
        print(json.dumps({"config": args.config, "P": P, "nq": int(Q.shape[0]), "k": k,
                          "entries_kept_frac": frac, "bytes_per_rank_unpruned": (P - 1) / P * Q.shape[0] * k * 8,
                          "bytes_per_rank_pruned": (P - 1) / P * Q.shape[0] * k * 8 * frac + Q.shape[0] * 8,
                          "same_result": same}), flush=True)


if __name__ == "__main__":
    main()
