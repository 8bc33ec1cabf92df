"""Summarise an ncu --set full report into markdown (key metrics per kernel)."""
import csv, subprocess, sys, io, collections
rep, title = sys.argv[1], sys.argv[2]
raw = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(raw)))
h = r[0]; units = r[1]; data = r[2:]
want = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "lts__t_bytes.sum",
        "sm__throughput.avg.pct_of_peak_sustained_elapsed", "gpu__compute_memory_throughput.avg.pct_of_peak_sustained_elapsed",
        "sm__warps_active.avg.pct_of_peak_sustained_active", "smsp__thread_inst_executed_per_inst_executed.ratio",
        "sm__inst_executed.sum", "smsp__inst_executed.avg.per_cycle_active", "launch__registers_per_thread",
        "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active", "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
        "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active", "l1tex__t_sector_hit_rate.pct", "lts__t_sector_hit_rate.pct",
        "sm__pipe_tc_cycles_active.avg.pct_of_peak_sustained_active", "sm__pipe_tensor_cycles_active.avg.pct_of_peak_sustained_active",
        "launch__grid_size", "launch__block_size"]
idx = {w: h.index(w) for w in want if w in h}
ki = h.index("Kernel Name")
out = ["# " + title, "", "ncu --set full --clock-control none --import-source on (one capture per kernel; replayed, so durations are cold-cache)", ""]
out.append("| kernel | " + " | ".join(w for w in idx) + " |")
out.append("|---|" + "---|" * len(idx))
for row in data:
    out.append("| " + row[ki].split("(")[0].replace("void ", "")[:40] + " | " + " | ".join(
        (row[i] + (" " + units[i] if units[i] else "")) for w, i in idx.items()) + " |")
print("\n".join(out))
