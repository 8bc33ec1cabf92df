"""Fig. 8's r (cache-conflict factor) on B200: ms per join for
r in {0.25 (paper), 0.5, 1, 2, 4} -- r * max_cur vs |Q| sets the minimum tile
split of the thread-per-query scan.  python tools/rfactor_sweep.py C1 C2 C3"""
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
        for r in (0.25, 0.5, 1.0, 2.0, 4.0, 8.0):
            ms = time_ms(lambda: sknn.join(dQ, dT, k, r_factor=r), 7)
            _, _, st = sknn.join(dQ, dT, k, r_factor=r, stats=True)
            print(json.dumps({"config": name, "r": r, "ms": ms, "pruned_pct": st["pruned_pct"],
                              "ms_sparse": st["ms_sparse"]}), flush=True)


if __name__ == "__main__":
    main()
