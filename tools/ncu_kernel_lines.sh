#!/bin/bash
# Per-source-line hot spots of one kernel (by name regex) in an ncu report:
#   tools/ncu_kernel_lines.sh rep.ncu-rep <kernel-regex> [n] [launch-skip]
rep=$1; k=$2; n=${3:-25}; skip=${4:-0}
ncu -i "$rep" --page source --csv --print-source cuda,sass -k "regex:$k" --launch-skip $skip --launch-count 1 2>&1 | python -c "
import csv,sys
out=[];f=None
for r in csv.reader(sys.stdin):
  if r and r[0]=='File Path': f=r[1].split('/')[-1]; continue
  if len(r)>8 and r[0].isdigit():
    try: out.append((int(r[4]),int(r[7]),f,r[0],r[1].strip()[:100]))
    except: pass
tot=sum(o[0] for o in out) or 1; ti=sum(o[1] for o in out) or 1
out.sort(reverse=True)
print('stall samples %d, warp inst %d' % (tot, ti))
for o in out[:$n]: print('%5.1f%% %5.1f%%  %s:%s  %s'%(100*o[0]/tot,100*o[1]/ti,o[2],o[3],o[4]))
"
