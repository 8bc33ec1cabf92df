"""Option sweep on the GPU: per-stage times and pruning for the C1-C5 workloads.

    python tools/sweep.py [--configs C2,C3] [--scale 1.0] [--reps 5] [--variants default,lloyd0,...]

Prints one JSON line per (config, variant): median ms_total over reps, the stage
split (CUDA events inside the library), % pruned, evaluations per query.
"""
import argparse
import json
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import datagen  # noqa: E402

VARIANTS = {
    "default": {},
    "lloyd0": {"lloyd_iters": 0},
    "lloyd1": {"lloyd_iters": 1},
    "lloyd4": {"lloyd_iters": 4},
    "thread": {"mapping": "thread"},
    "sparse": {"force_path": "sparse"},
    "partial": {"force_path": "partial"},
    "dense": {"force_path": "dense"},
    "tau4": {"dense_threshold": 4.0},
    "tau25": {"dense_threshold": 0.25},
    "tau50": {"dense_threshold": 0.5},
    "tau75": {"dense_threshold": 0.75},
    "tau95": {"dense_threshold": 0.95},
    "tau99": {"dense_threshold": 0.99},
    "warp": {"mapping": "warp"},
    "cl_half": {"_cl": 0.5},
    "cl_double": {"_cl": 2.0},
    "cl_0.7": {"_cl": 0.7},
    "cl_1.4": {"_cl": 1.4},
    "fullassign": {"_env": ("SKNN_ASSIGN", "full")},
    "walkassign": {"_env": ("SKNN_ASSIGN", "walk")},
    "tcassign": {"_env": ("SKNN_ASSIGN", "tc")},
    "entries256": {"_env": ("SKNN_WALK_ENTRIES", "256")},
    "paperseed": {"_env": ("SKNN_SEEDING", "paper")},
    "topk_reg": {"_env": ("SKNN_TOPK", "reg")},
    "topk_smem": {"_env": ("SKNN_TOPK", "smem")},
    "full_lloyd4": {"_env": ("SKNN_ASSIGN", "full"), "lloyd_iters": 4},
}


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--configs", default="C1,C2,C3,C3int")
    ap.add_argument("--scale", type=float, default=1.0)
    ap.add_argument("--reps", type=int, default=5)
    ap.add_argument("--variants", default="default")
    ap.add_argument("--k", type=int, default=0, help="override the config's k (k sweep, Fig. 10 / Table V)")
    args = ap.parse_args()
    import torch
    import paper_conf_icde_chends17_b200 as sknn
    for name in args.configs.split(","):
        Q, T, k, sj = datagen.workload(name, args.scale)
        k = args.k or k
        dQ = torch.from_numpy(Q).cuda()
        dT = dQ if sj else torch.from_numpy(T).cuda()
        nq, nt = Q.shape[0], T.shape[0]
        flush = torch.empty(128 * 1024 * 1024, dtype=torch.float32, device="cuda")
        for vname in args.variants.split(","):
            if vname.startswith("env:"):  # ad-hoc variant: env:NAME=VALUE[+NAME2=VALUE2...]
                v = {"_env": [tuple(kv.split("=")) for kv in vname[4:].split("+")]}
            else:
                v = dict(VARIANTS[vname])
            env = v.pop("_env", None)
            cl = v.pop("_cl", None)
            if cl:
                v["n_clusters_t"] = int(3 * np.sqrt(nt) * cl)
                v["n_clusters_q"] = int(3 * np.sqrt(nq) * cl)
            if env and isinstance(env, tuple):
                env = [env]
            for n_, v_ in env or []:
                os.environ[n_] = v_
            res = []
            for r in range(args.reps + 2):
                flush.zero_()
                _, _, st = sknn.join(dQ, dT, k, stats=True, **v)
                if r >= 2:
                    res.append(st)
            for n_, _ in env or []:
                del os.environ[n_]
            ms = [x["ms_total"] for x in res]
            med = res[int(np.argsort(ms)[len(ms) // 2])]
            out = {"config": name, "variant": vname, "nq": nq, "nt": nt, "k": k, "ms_total": float(np.median(ms)),
                   "ms_min": float(np.min(ms)), "queries_per_s": nq / (np.median(ms) / 1000.0),
                   "pruned_pct": med["pruned_pct"], "evals_per_query": med["dist_evals"] / nq,
                   "cand_per_qcluster": med["cand_pairs"] / max(1, med["mq"]), "center_evals_per_query": med["center_evals"] / nq,
                   "inserts_per_query": med.get("topk_inserts", 0) / nq,
                   "stages": {k2: round(med[k2], 4) for k2 in ("ms_build_t", "ms_build_q", "ms_level1", "ms_dense", "ms_sparse")},
                   "dense_pairs": med["dense_pairs"], "evals_dense": med["dist_evals_dense"], "recompute": med["dist_recompute"],
                   "mq": med["mq"], "mt": med["mt"], "mapping": med["mapping_used"], "launches": med["kernel_launches"]}
            print(json.dumps(out), flush=True)


if __name__ == "__main__":
    main()
