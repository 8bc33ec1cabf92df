"""Per-source-line hot spots of one kernel from an ncu report: python tools/ncu_lines.py rep.ncu-rep [n]"""
import csv
import io
import subprocess
import sys

rep = sys.argv[1]
n = int(sys.argv[2]) if len(sys.argv) > 2 else 40
raw = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
out, f = [], None
for r in csv.reader(io.StringIO(raw)):
    if r and r[0] == "File Path":
        f = r[1].split("/")[-1]
        continue
    if len(r) > 8 and r[0].isdigit():
        try:
            out.append((int(r[4]), int(r[7]), f, r[0], r[1].strip()[:90]))
        except ValueError:
            pass
tot = sum(o[0] for o in out) or 1
ti = sum(o[1] for o in out) or 1
out.sort(reverse=True)
print(f"stall samples {tot}, warp instructions {ti}")
print("samples  inst   where")
for o in out[:n]:
    print("%5.1f%% %5.1f%%  %s:%s  %s" % (100 * o[0] / tot, 100 * o[1] / ti, o[2], o[3], o[4]))
