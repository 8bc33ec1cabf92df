"""Window-union estimate for a warp-cooperative level-2 scan (design study, GPU box).

python tools/union_sim.py C2 [scale]

For every query q and candidate target cluster tc of its query cluster (level-1 output
of the library), the Alg. 2 window under the FINAL theta (q's true k-th distance) is
W(q, tc) = #{t in tc : |d(q, c_tc) - d(t, c_tc)| <= theta_q}. A warp that walks the
union of its 32 lanes' windows evaluates U(tile, tc) = #{t : dt in [min(dq - theta),
max(dq + theta)]} members for every active lane. Reports sum W (per-thread scan) against
32 * sum U for tiles made of 32 consecutive members in radius order and in a spatial
(principal-axis) order."""
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
    dQ = dT if sj else torch.from_numpy(Q).cuda()
    _, dist = sknn.join(dQ, dT, k)
    theta = dist[:, -1].cpu().numpy().astype(np.float64)
    ix = sknn.build(dT)
    ex = ix.export()
    dbg = ix.debug_level1(dQ, k)
    off, tdist, cent = ex["off"], ex["dist"].astype(np.float64), ex["centers"][:, : Q.shape[1]].astype(np.float64)
    mq = dbg["mq"]
    qcl = dbg["q_cluster"]
    Qd = Q.astype(np.float64)
    # per query cluster: members, radius order and a principal-axis order
    order = np.argsort(qcl, kind="stable")
    qoff = np.concatenate([[0], np.cumsum(np.bincount(qcl, minlength=mq))])
    tiles_r, tiles_s = [], []
    for c in range(mq):
        mem = order[qoff[c]:qoff[c + 1]]
        if len(mem) == 0:
            continue
        X = Qd[mem]
        mu = X.mean(0)
        r = np.sqrt(((X - mu) ** 2).sum(1))
        mr = mem[np.argsort(-r, kind="stable")]
        Xc = X - mu
        if len(mem) > 1:
            _, _, vt = np.linalg.svd(Xc, full_matrices=False)
            proj = Xc @ vt[0]
        else:
            proj = np.zeros(1)
        ms = mem[np.argsort(proj, kind="stable")]
        for i in range(0, len(mem), 32):
            tiles_r.append((c, mr[i:i + 32]))
            tiles_s.append((c, ms[i:i + 32]))
    cand = dbg["cand"]
    cc = dbg["cand_count"]
    res = {}
    for label, tiles in (("radius", tiles_r), ("spatial", tiles_s)):
        W = 0.0
        U = 0.0
        Ulanes = 0.0
        for c, q in tiles:
            th = theta[q]
            for tc in cand[c, : cc[c]]:
                lo, hi = off[tc], off[tc + 1]
                seg = -tdist[lo:hi]  # ascending
                dq = np.sqrt(((Qd[q] - cent[tc]) ** 2).sum(1))
                a = np.searchsorted(seg, -(dq + th), side="left")
                b = np.searchsorted(seg, -(dq - th), side="right")
                w = np.maximum(b - a, 0)
                act = w > 0
                if not act.any():
                    continue
                W += w.sum()
                u = b[act].max() - a[act].min()
                U += u * 32
                Ulanes += u * act.sum()
        res[label] = (W, U, Ulanes)
        nq = Q.shape[0]
        print(f"{name} {label:8s}: per-thread evals/query {W / nq:8.1f}  union evals/query (32 lanes) {U / nq:8.1f} "
              f"(active lanes {Ulanes / nq:8.1f})  waste x{U / max(W, 1):.2f}")


if __name__ == "__main__":
    main()
