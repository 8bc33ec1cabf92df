# source-able: reduce <report-base> -> raw CSV (gz), markdown summary, per-line hot spots;
# the .ncu-rep is deleted unless its basename is listed in $KEEP (gpurun copies back <= 64 MiB)
reduce() {
  local r=$1
  [ -f $r.ncu-rep ] || return
  ncu -i $r.ncu-rep --page raw --csv > $r.raw.csv 2>/dev/null
  python profiles/ncu_summary.py $r.ncu-rep "$(basename $r)" > $r.md 2>/dev/null
  python tools/ncu_lines.py $r.ncu-rep 40 > $r.lines.txt 2>/dev/null
  gzip -f $r.raw.csv
  case " $KEEP " in *" $(basename $r) "*) ;; *) rm -f $r.ncu-rep ;; esac
}
