"""Run a few joins of one workload (for ncu captures): python tools/run_one.py C4 [scale] [reps] [opt=v ...] [knn_k=k]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import datagen  # noqa: E402


def main():
    name = sys.argv[1]
    scale = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
    reps = int(sys.argv[3]) if len(sys.argv) > 3 else 1
    opts = {}
    for kv in sys.argv[4:]:
        k, v = kv.split("=")
        opts[k] = int(v) if v.lstrip("-").isdigit() else v
    import torch
    import paper_conf_icde_chends17_b200 as sknn
    Q, T, k, sj = datagen.workload(name, scale)
    k = int(opts.pop("knn_k", k))  # knn_k=<k> overrides the config's k
    dQ = torch.from_numpy(Q).cuda()
    dT = dQ if sj else torch.from_numpy(T).cuda()
    for _ in range(reps):
        _, _, st = sknn.join(dQ, dT, k, stats=True, **opts)
    torch.cuda.synchronize()
    print({key: st[key] for key in ("ms_total", "ms_build_t", "ms_build_q", "ms_level1", "ms_dense", "ms_sparse",
                                     "pruned_pct", "dist_evals_dense", "dist_recompute", "dense_pairs")})


if __name__ == "__main__":
    main()
