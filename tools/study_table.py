"""Format gpurun_out/study/{ksweep,ablation}.jsonl (tools/study.sh) as markdown tables:
python tools/study_table.py gpurun_out/study > profiles/r01_study.md"""
import json
import os
import sys


def load(path):
    out = []
    for line in open(path):
        try:
            out.append(json.loads(line))
        except ValueError:
            pass
    return out


def main():
    d = sys.argv[1]
    ks = load(os.path.join(d, "ksweep.jsonl"))
    ab = load(os.path.join(d, "ablation.jsonl"))
    print("# r01 studies on synthetic data (one B200; `tools/study.sh`, `tools/sweep.py`: median of 3 joins after 2 "
          "warm-ups, L2 flushed)\n")
    print("## k sweep, full vs partial level-2 filter (paper Fig. 10 / Table V, P:L805-821)\n")
    print("`full` = the full filter (running theta, kNearests; dense tiles off; k <= 96 per-thread heap, k > 96 the "
          "warp-per-query thresholded buffer of k_scan_bigk), `partial` = SKNN_PATH_PARTIAL (theta fixed at the level-1 "
          "UB, survivor buffer, k-selection). C2 at k = 512: the survivor buffer exceeds half the free HBM, so "
          "`partial` counted its windows and then fell back to the full filter (identical counts). On B200 the full "
          "filter wins every case, so auto never picks the partial filter (DESIGN.md reading R13).\n")
    print("| config | k | k/d | filter | ms / join | % pruned | evals / query |")
    print("|---|---|---|---|---|---|---|")
    dims = {"C2": 4, "C3": 28}
    for r in ks:
        v = "full" if r["variant"] == "sparse" else "partial"
        print("| %s | %d | %.1f | %s | %.3f | %.3f | %.0f |" % (r["config"], r["k"], r["k"] / dims.get(r["config"], 1), v,
                                                             r["ms_total"], r["pruned_pct"], r["evals_per_query"]))
    print("\n## Ablations (paper Fig. 11 #landmarks, Fig. 12 / Table IV threads per query, Lloyd / seeding)\n")
    print("`cl_x` = x * 3*sqrt(n) clusters (clamped to 8192); `thread` / `warp` = query-level vs warp-per-query "
          "mapping; `lloyd0/1` = Lloyd iterations (default 2); `paperseed` = the paper's sampler only (no D^2 seeding "
          "half); `sparse` = elastic switch off. `env:SKNN_WALK=lane` only affects the runtime-k scan (the configs' k "
          "run the compile-time-k union walk), so it equals the default here.\n")
    print("| config | variant | ms / join | % pruned | evals / query | clusters | mapping | build / level-1 / dense / sparse ms |")
    print("|---|---|---|---|---|---|---|---|")
    for r in ab:
        st = r["stages"]
        print("| %s | %s | %.3f | %.3f | %.0f | %d | %s | %.3f / %.3f / %.3f / %.3f |" % (
            r["config"], r["variant"], r["ms_total"], r["pruned_pct"], r["evals_per_query"], r["mq"],
            "thread" if r["mapping"] == 1 else "warp", st["ms_build_t"] + st["ms_build_q"], st["ms_level1"],
            st["ms_dense"], st["ms_sparse"]))


if __name__ == "__main__":
    main()
