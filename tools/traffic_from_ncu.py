"""profiles/traffic.json from ncu --set full raw CSVs (one capture per kernel):
dram__bytes_read.sum + dram__bytes_write.sum per launch, keyed by config and
kernel, for bench.py's roofline `traffic` field.

    python tools/traffic_from_ncu.py gpurun_out/r02final [profiles/traffic.json]
"""
import csv
import glob
import gzip
import io
import json
import os
import sys

SCALE = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def main():
    src = sys.argv[1]
    dst = sys.argv[2] if len(sys.argv) > 2 else os.path.join(os.path.dirname(__file__), "..", "profiles", "traffic.json")
    out = {"_about": "dram__bytes_read.sum + dram__bytes_write.sum per launch of the config's kernel, ncu --set full "
                     "--clock-control none (one capture, cold cache); source: %s" % os.path.basename(src.rstrip("/"))}
    for f in sorted(glob.glob(os.path.join(src, "*.raw.csv.gz"))):
        name = os.path.basename(f)[:-len(".raw.csv.gz")]
        if "_" not in name or not name[:2].startswith("c"):
            continue
        cfg, kernel = name.split("_", 1)
        kernel = kernel.replace("_alldense", "")
        rows = list(csv.reader(io.StringIO(gzip.open(f, "rt").read())))
        h, units, data = rows[0], rows[1], rows[2:]
        if not data:
            continue
        tot = 0.0
        for m in ("dram__bytes_read.sum", "dram__bytes_write.sum"):
            i = h.index(m)
            tot += float(data[0][i].replace(",", "")) * SCALE.get(units[i], 1.0)
        key = kernel.replace("k_dense_exact", "k_dense")
        if name.endswith("_alldense"):
            key += "_alldense"
        out.setdefault(cfg.upper(), {})[key] = tot
    with open(dst, "w") as fh:
        json.dump(out, fh, indent=1, sort_keys=True)
    print(json.dumps(out, indent=1, sort_keys=True))


if __name__ == "__main__":
    main()
