"""Seeding A/B (reading R9): the paper's landmark sampler alone
(SKNN_SEEDING=paper) vs the D^2 split (SKNN_SEEDING=d2) on named workloads
(C1-C5, C3int, and the ablation shapes G<d> / K<d> of datagen.workload).
ms per join = median of CUDA-event timings (graph replay), % pruned from stats.

    python tools/seed_ab.py C3 C5 G16 K28 ...
"""
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
sys.path.insert(0, os.path.dirname(os.path.abspath(__file__)))

import datagen  # noqa: E402


def main():
    import torch
    import paper_conf_icde_chends17_b200 as sknn
    from tools_timing import time_ms
    for name in sys.argv[1:]:
        Q, T, k, sj = datagen.workload(name)
        dQ = torch.from_numpy(Q).cuda()
        dT = dQ if sj else torch.from_numpy(T).cuda()
        for sd in ("paper", "d2"):
            os.environ["SKNN_SEEDING"] = sd
            ms = time_ms(lambda: sknn.join(dQ, dT, k, use_graph=-1), 5)
            _, _, st = sknn.join(dQ, dT, k, stats=True)
            print(json.dumps({"config": name, "d": int(Q.shape[1]), "seeding": sd, "ms": ms,
                              "pruned_pct": st["pruned_pct"], "ms_build": st["ms_build_t"] + st["ms_build_q"]}),
                  flush=True)
        os.environ.pop("SKNN_SEEDING", None)
        del dQ, dT
        torch.cuda.empty_cache()


if __name__ == "__main__":
    main()
