"""Time sknn_merge_partials at C5 target-sharded sizes (the
HBM-gate kernel at P = 8): P sorted partial lists of k (d2, global idx) per
query, nq queries -> the k smallest per query. Synthetic, seeded, built on
the device (the partials' values do not change the merge's work).

    python tools/merge_bench.py [--nq 4000000] [--k 32] [--P 8] [--reps 5]

Prints one JSON line per P: ms per merge (CUDA events on the launching
stream, after a warm-up) and the algorithmic HBM bytes (8 k nq P read +
8 k nq written) / time against MEASURED_PEAKS.json's HBM figure.
"""
import argparse
import json
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--nq", type=int, default=4_000_000)
    ap.add_argument("--k", type=int, default=32)
    ap.add_argument("--P", default="8")
    ap.add_argument("--reps", type=int, default=5)
    args = ap.parse_args()
    import torch
    import paper_conf_icde_chends17_b200 as sknn
    peak = None
    pp = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(pp):
        peak = json.load(open(pp)).get("hbm_gbs")
    g = torch.Generator(device="cuda")
    g.manual_seed(7)
    for P in [int(x) for x in args.P.split(",")]:
        nq, k = args.nq, args.k
        d2 = torch.rand((P, nq, k), device="cuda", generator=g) * 1000.0
        d2 = d2.round()  # integer-valued: ties across lists exercise the index order
        d2, _ = torch.sort(d2, dim=2)
        # global indices: list p holds targets of shard p; ascending within equal d2
        idx = (torch.arange(k, device="cuda", dtype=torch.int32)[None, None, :] +
               torch.arange(P, device="cuda", dtype=torch.int32)[:, None, None] * 1_000_000 +
               (torch.arange(nq, device="cuda", dtype=torch.int32)[None, :, None] % 997) * k)
        oi = torch.empty((nq, k), dtype=torch.int32, device="cuda")
        od = torch.empty((nq, k), dtype=torch.float32, device="cuda")
        s = torch.cuda.current_stream()
        sknn.merge_partials(idx, d2, k, out=(oi, od), out_squared=True, stream=s)
        torch.cuda.synchronize()
        ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.reps)]
        for a, b in ev:
            a.record(s)
            sknn.merge_partials(idx, d2, k, out=(oi, od), out_squared=True, stream=s)
            b.record(s)
        torch.cuda.synchronize()
        ms = sorted(a.elapsed_time(b) for a, b in ev)[len(ev) // 2]
        byts = 8.0 * k * nq * P + 8.0 * k * nq
        gbs = byts / (ms / 1e3) / 1e9
        # spot check against torch (sort of the concatenated keys)
        q = torch.randint(0, nq, (256,), device="cuda", generator=g)
        keys = (d2[:, q, :].double() * 2**32 + idx[:, q, :].double()).permute(1, 0, 2).reshape(256, -1)
        want = torch.sort(keys, dim=1).values[:, :k]
        got = od[q].double() * 2**32 + oi[q].double()
        ok = bool(torch.equal(torch.round(want), torch.round(got)))
        print(json.dumps({"P": P, "nq": nq, "k": k, "ms": ms, "bytes": byts, "gbs": gbs,
                          "hbm_peak_gbs": peak, "frac": gbs / peak if peak else None, "spot_check": ok}), flush=True)
        del d2, idx, oi, od


if __name__ == "__main__":
    main()
