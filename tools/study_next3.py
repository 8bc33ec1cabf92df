"""Summarise a tools/paper_study_ncu.sh run (NEXT-3) as markdown: the
three-arm timing table (Sweet / basic KNN-TI / cuBLAS brute force) and the
Table IV analogue (pruned %, warp efficiency of the level-2 scan kernel).

    python tools/study_next3.py gpurun_out/<tag>
"""
import csv
import io
import json
import os
import sys


def ncu_rows(path):
    lines = [l for l in open(path) if l.startswith('"')]
    out = {}
    for r in csv.DictReader(io.StringIO("".join(lines))):
        kn = r["Kernel Name"].split("(")[0].replace("void ", "")
        d = out.setdefault(kn, {})
        d[r["Metric Name"]] = float(r["Metric Value"].replace(",", ""))
    return out


def main():
    base = sys.argv[1]
    recs = [json.loads(l) for l in open(os.path.join(base, "study.jsonl")) if l.startswith("{")]
    by = {}
    for r in recs:
        by.setdefault(r["config"], {})[r["arm"]] = r
    print("| Config | Sweet ms / join | basic KNN-TI ms (same queries) | cuBLAS brute force ms (same queries) | "
          "Sweet vs basic | Sweet vs cuBLAS | pruned % Sweet / basic |")
    print("|---|---|---|---|---|---|---|")
    for c, a in by.items():
        sw, ba, ge = a.get("sweet"), a.get("basic"), a.get("gemm")
        sw_ms = sw["ms"]
        # like-for-like: the sample's Sweet time when basic ran on a sample
        sw_b = ba.get("ms_sweet_same_sample", sw_ms) if ba else None
        sp_b = ba["ms"] / sw_b if ba else None
        # gemm per query x nq vs the full Sweet join (brute force is linear in nq)
        ge_full = ge["ms"] * sw["nq_timed"] / ge["nq_timed"] if ge else None
        print("| %s | %.3f | %s | %s | %s | %s | %.3f / %s |" % (
            c, sw_ms,
            ("%.2f (%d q)" % (ba["ms"], ba["nq_timed"])) if ba else "-",
            ("%.1f (%d q) -> %.1f full" % (ge["ms"], ge["nq_timed"], ge_full)) if ge else "-",
            ("%.1fx" % sp_b) if ba else "-",
            ("%.0fx" % (ge_full / sw_ms)) if ge else "-",
            sw["pruned_pct"], ("%.3f" % ba["pruned_pct"]) if ba else "-"))
    print()
    print("| Config | scan kernel (Sweet) | warp efficiency Sweet | basic KNN-TI warp efficiency | "
          "scan ms Sweet / basic (ncu) | instructions Sweet / basic |")
    print("|---|---|---|---|---|---|")
    for c in ("C1", "C2", "C3", "C4", "C5"):
        fa, fb = (os.path.join(base, "warpeff_%s_%s.csv" % (c, m)) for m in ("auto", "basic"))
        if not (os.path.exists(fa) and os.path.exists(fb)):
            continue
        ra, rb = ncu_rows(fa), ncu_rows(fb)
        ka = [k for k in ra if k.startswith("k_scan")]
        kb = [k for k in rb if k.startswith("k_scan")]
        if not ka or not kb:
            continue
        a, b = ra[ka[0]], rb[kb[0]]
        r = "smsp__thread_inst_executed_per_inst_executed.ratio"
        print("| %s | %s | %.1f%% | %.1f%% | %.3f / %.3f | %.3g / %.3g |" % (
            c, ka[0], 100 * a[r] / 32, 100 * b[r] / 32, a["gpu__time_duration.sum"] / 1e6,
            b["gpu__time_duration.sum"] / 1e6, a["smsp__inst_executed.sum"], b["smsp__inst_executed.sum"]))


if __name__ == "__main__":
    main()
