"""Live kernel timeline of one join (CUPTI via torch.profiler): per-kernel durations and the idle
gaps between consecutive kernels. python tools/timeline.py C2 [scale] [reps]"""
import os
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)
import datagen  # noqa: E402


def main():
    name = sys.argv[1]
    scale = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
    reps = int(sys.argv[3]) if len(sys.argv) > 3 else 3
    import torch
    from torch.profiler import ProfilerActivity, profile
    import paper_conf_icde_chends17_b200 as sknn
    Q, T, k, sj = datagen.workload(name, scale)
    dQ = torch.from_numpy(Q).cuda()
    dT = dQ if sj else torch.from_numpy(T).cuda()
    for _ in range(3):
        sknn.join(dQ, dT, k)
    torch.cuda.synchronize()
    with profile(activities=[ProfilerActivity.CUDA]) as prof:
        for _ in range(reps):
            sknn.join(dQ, dT, k)
        torch.cuda.synchronize()
    evs = [e for e in prof.events() if e.device_type == torch.autograd.DeviceType.CUDA]
    evs.sort(key=lambda e: e.time_range.start)
    # every join launches the same sequence: take the last len/reps events
    n = len(evs) // reps
    j = evs[-n:]
    t0 = j[0].time_range.start
    busy = 0.0
    print(f"{'start_us':>9} {'dur_us':>8} {'gap_us':>7}  kernel")
    prev_end = None
    for e in j:
        s, d = e.time_range.start, e.time_range.end - e.time_range.start
        gap = 0.0 if prev_end is None else s - prev_end
        busy += d
        print(f"{s - t0:9.1f} {d:8.1f} {gap:7.1f}  {e.name[:70]}")
        prev_end = e.time_range.end
    span = j[-1].time_range.end - t0
    print(f"span {span:.1f} us, kernel busy {busy:.1f} us, idle {span - busy:.1f} us, {len(j)} launches")


if __name__ == "__main__":
    main()
