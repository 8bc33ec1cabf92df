import sys, os, json
sys.path.insert(0, os.getcwd())
import torch, datagen
import paper_conf_icde_chends17_b200 as sknn
Q, T, k, sj = datagen.workload("C4")
dT = torch.from_numpy(T).cuda()
for P in (1, 2, 8):
    for r in range(min(P, 2)):
        lo, hi = r * Q.shape[0] // P, (r + 1) * Q.shape[0] // P
        qr = torch.from_numpy(Q[lo:hi]).cuda()
        for opts in ({}, {"n_clusters_q": 3000}, {"lloyd_iters": 4}):
            sknn.join(qr, dT, k)
            _, _, st = sknn.join(qr, dT, k, stats=True, **opts)
            print(P, r, opts, {kk: (round(v, 3) if isinstance(v, float) else v) for kk, v in st.items() if kk in ("ms_total","ms_build_q","ms_build_t","ms_level1","ms_dense","ms_sparse","mq","mt","dense_pairs","cand_pairs","dist_evals_sparse","dist_evals_dense","center_evals")}, flush=True)
