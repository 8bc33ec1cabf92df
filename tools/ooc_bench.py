"""Out-of-core sknn_query (NEXT-4): host queries and host outputs streamed
through the device in batches against a resident index; serial batches
(SKNN_OOC_SERIAL=1) vs the overlapped two-stream pipeline, pageable and
page-locked host buffers. Wall time per call (host clock around the call,
which returns with the results in host memory), median of reps.

    python tools/ooc_bench.py [--config C5] [--batch 500000] [--reps 3]
"""
import argparse
import json
import os
import statistics
import sys
import time

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import numpy as np  # noqa: E402

import datagen  # noqa: E402


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--config", default="C5")
    ap.add_argument("--batch", type=int, default=500_000)
    ap.add_argument("--reps", type=int, default=3)
    args = ap.parse_args()
    import torch
    import paper_conf_icde_chends17_b200 as sknn
    Q, T, k, sj = datagen.workload(args.config)
    ix = sknn.build(torch.from_numpy(T).cuda())
    nq = Q.shape[0]
    pq = torch.from_numpy(Q).pin_memory()
    pi = torch.empty((nq, k), dtype=torch.int32).pin_memory()
    pd = torch.empty((nq, k), dtype=torch.float32).pin_memory()
    ref = None
    for mode in ("serial", "overlap"):
        for mem in ("pageable", "pinned"):
            if mode == "serial":
                os.environ["SKNN_OOC_SERIAL"] = "1"
            else:
                os.environ.pop("SKNN_OOC_SERIAL", None)
            ts = []
            for _ in range(args.reps + 1):
                torch.cuda.synchronize()
                t0 = time.perf_counter()
                if mem == "pageable":
                    i, d = ix.query(Q, k, query_batch=args.batch)
                else:
                    ix.query(pq, k, query_batch=args.batch, out=(pi, pd))
                    i, d = pi.numpy(), pd.numpy()
                ts.append((time.perf_counter() - t0) * 1e3)
            ok = True
            if ref is None:
                ref = (np.array(i), np.array(d))
            else:
                ok = bool(np.array_equal(ref[0], i) and np.array_equal(ref[1].view(np.uint32), np.asarray(d).view(np.uint32)))
            ms = statistics.median(ts[1:])
            print(json.dumps({"config": args.config, "nq": nq, "k": k, "batch": args.batch, "mode": mode, "host_mem": mem,
                              "ms": ms, "queries_per_s": nq / (ms / 1e3), "same_result": ok,
                              "h2d_bytes": 4 * Q.size, "d2h_bytes": 8 * nq * k}), flush=True)
    os.environ.pop("SKNN_OOC_SERIAL", None)
    ix.close()


if __name__ == "__main__":
    main()
