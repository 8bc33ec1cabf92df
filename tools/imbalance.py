"""Per-query-cluster work estimate after level-1 (load-balance analysis of the scan).

python tools/imbalance.py G32 [scale]
work(qc) = |qc| * sum over candidate target clusters of their sizes (an upper bound on
member visits); prints the heaviest clusters against the mean per warp tile."""
import os
import sys

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import datagen  # noqa: E402


def main():
    name = sys.argv[1]
    scale = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
    import torch
    import paper_conf_icde_chends17_b200 as sknn
    Q, T, k, sj = datagen.workload(name, scale)
    dT = torch.from_numpy(T).cuda()
    idx = sknn.build(dT)
    inf = idx.info()
    dbg = idx.debug_level1(torch.from_numpy(Q).cuda(), k)
    mq = dbg["mq"]
    qsz = np.bincount(dbg["q_cluster"], minlength=mq)
    ex = idx.export()
    tsz = np.diff(ex["off"])
    cc = dbg["cand_count"]
    reach = np.array([tsz[dbg["cand"][i, : cc[i]]].sum() for i in range(mq)], dtype=np.float64)
    tiles = np.ceil(qsz / 32.0)
    per_tile = reach  # member visits per lane ~ reach
    total = (tiles * per_tile).sum()
    order = np.argsort(-per_tile)
    print(f"{name}: mq={mq} mt={inf['mt']} tiles={int(tiles.sum())} mean cand={cc.mean():.1f} max cand={cc.max()}")
    print(f"mean reach/tile={total / tiles.sum():.0f}  max reach/tile={per_tile.max():.0f}  "
          f"ratio={per_tile.max() / (total / tiles.sum()):.1f}")
    print(" qc   |qc|  cand   ub        reach")
    for i in order[:12]:
        print(f"{i:5d} {qsz[i]:5d} {cc[i]:5d} {dbg['ub'][i]:9.3f} {per_tile[i]:9.0f}")
    print("ub quantiles", np.quantile(dbg["ub"], [0.0, 0.5, 0.9, 0.99, 1.0]))
    print("target radius quantiles", np.quantile(ex["radius"], [0.0, 0.5, 0.9, 0.99, 1.0]))
    print("target size quantiles", np.quantile(tsz, [0.0, 0.5, 0.9, 0.99, 1.0]))


if __name__ == "__main__":
    main()
