"""Summarise an `ncu --metrics gpu__time_duration.sum --csv` launch list into a markdown table.

python tools/launch_summary.py launches.csv "title" [joins]
Launch counts and times are divided by `joins` (the number of joins the profiled command ran) so
the table reads per join."""
import collections
import csv
import sys


def main():
    path, title = sys.argv[1], sys.argv[2]
    rows = [r for r in csv.DictReader(l for l in open(path) if not l.startswith("==")) if r.get("Metric Name") == "gpu__time_duration.sum"]
    ids = sorted({int(r["ID"]) for r in rows})
    joins = int(sys.argv[3]) if len(sys.argv) > 3 else 1
    keep = set(ids)
    agg = collections.OrderedDict()
    for r in rows:
        if int(r["ID"]) not in keep:
            continue
        name = r["Kernel Name"].split("(")[0].replace("void ", "")
        v = float(r["Metric Value"].replace(",", ""))
        if r["Metric Unit"] in ("nsecond", "ns"):
            v /= 1000.0
        elif r["Metric Unit"] in ("msecond", "ms"):
            v *= 1000.0
        c, t = agg.get(name, (0, 0.0))
        agg[name] = (c + 1, t + v)
    tot = sum(t for _, t in agg.values())
    print(f"# {title}\n")
    print("| kernel | launches/join | us/join | share |\n|---|---|---|---|")
    for name, (c, t) in sorted(agg.items(), key=lambda kv: -kv[1][1]):
        print(f"| {name} | {c / joins:g} | {t / joins:.1f} | {100 * t / tot:.1f}% |")
    print(f"| **total** | {sum(c for c, _ in agg.values()) / joins:g} | {tot / joins:.1f} | 100% |")


if __name__ == "__main__":
    main()
