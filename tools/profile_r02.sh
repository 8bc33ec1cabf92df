#!/bin/bash
# Round-2 ncu evidence pass (run under gpurun, one GPU):
#   tools/profile_r02.sh <tag> [what...]
# what: fma | c4 | c5 | c2 | merge   (default: all)
# -> gpurun_out/<tag>/: fma_peak.json, ncu --set full reports (*.ncu-rep) of
#    the kernels SURVEY §8(d.4) names, one capture per kernel (-c 1).
tag=$1; shift
what=${@:-fma c4 c5 c2 merge}
out=gpurun_out/$tag; mkdir -p $out
python -c "import __graft_entry__ as g; g.build()" || exit 1
NCU="ncu --set full --import-source on --clock-control none -c 1"
# gpurun copies back <= 64 MiB: every report is reduced on the box to its raw
# metrics (CSV), a markdown summary and its per-line hot spots; only reports
# named in KEEP stay as .ncu-rep
KEEP=${KEEP:-"c4_k_dense"}
reduce() {  # reduce <report-base>
  local r=$1
  [ -f $r.ncu-rep ] || return
  ncu -i $r.ncu-rep --page raw --csv > $r.raw.csv 2>/dev/null
  python profiles/ncu_summary.py $r.ncu-rep "$(basename $r)" > $r.md 2>/dev/null
  python tools/ncu_lines.py $r.ncu-rep 40 > $r.lines.txt 2>/dev/null
  gzip -f $r.raw.csv
  case " $KEEP " in *" $(basename $r) "*) ;; *) rm -f $r.ncu-rep ;; esac
}
for w in $what; do
  case $w in
  fma)
    nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/fma_peak tools/fma_peak.cu && /tmp/fma_peak > $out/fma_peak.json
    ;;
  c4)
    for kn in k_dense k_scan_wpq k_level1 k_assign_tc k_scatter_keys k_gather_side; do
      timeout 900 $NCU -k regex:"^${kn}\$" -o $out/c4_$kn python tools/run_one.py C4 > $out/c4_$kn.txt 2>&1
      reduce $out/c4_$kn
    done
    ;;
  c5)
    for kn in k_scan_tpq k_level1 k_assign_tc k_scatter_keys k_gather_side k_merge_split; do
      timeout 900 $NCU -k regex:"^${kn}\$" -o $out/c5_$kn python tools/run_one.py C5 > $out/c5_$kn.txt 2>&1
      reduce $out/c5_$kn
    done
    ;;
  c2)
    timeout 600 $NCU -k regex:"^k_scan_tpq\$" -o $out/c2_k_scan_tpq python tools/run_one.py C2 2 > $out/c2_scan.txt 2>&1
    reduce $out/c2_k_scan_tpq
    timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $out/launches_c2.csv \
      python bench.py --steps 2 --warmup 3 --no-cpu-baseline > $out/launches_c2.txt 2>&1
    ;;
  merge)
    timeout 900 python tools/merge_bench.py > $out/merge_bench.jsonl 2>&1
    timeout 900 $NCU -k regex:"^k_merge" -o $out/merge_p8 python tools/merge_bench.py --reps 1 > $out/merge_ncu.txt 2>&1
    reduce $out/merge_p8
    ;;
  esac
done
ls -la $out
