"""One C4 query-row slice join (rank r of P): python tools/diag_c4_slice1.py P r [opt=v ...]"""
import os
import sys
sys.path.insert(0, os.getcwd())
import torch  # noqa: E402
import datagen  # noqa: E402
import paper_conf_icde_chends17_b200 as sknn  # noqa: E402
P, r = int(sys.argv[1]), int(sys.argv[2])
opts = {kv.split("=")[0]: int(kv.split("=")[1]) for kv in sys.argv[3:]}
Q, T, k, sj = datagen.workload("C4")
lo, hi = r * Q.shape[0] // P, (r + 1) * Q.shape[0] // P
qr = torch.from_numpy(Q[lo:hi]).cuda()
dT = torch.from_numpy(T).cuda()
_, _, st = sknn.join(qr, dT, k, stats=True, **opts)
print({kk: v for kk, v in st.items() if kk.startswith("ms_") or kk in ("mq", "dist_evals_sparse", "center_evals")})
