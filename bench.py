#!/usr/bin/env python
"""Benchmark of the B200-native Sweet KNN join (one JSON line on rank 0).

    python bench.py [--gpus N] [--steps K] [--warmup W] [--config C2]
                    [--mode query|target] [--exchange all_to_all|all_gather]
                    [--impl reference]

A step is one whole exact KNN join (all SURVEY §8(a) rows: clustering both
sides, level-1 calUB + groupFilter + elastic switch, dense tiles, level-2
filtered scan fused with top-k, result write; multi-GPU: the exchange and the
merge) on one workload, inputs resident in HBM. The default workload is
BASELINE.json configs[1] = C2, the 3D-road-network-shaped self-join (434,874 x
4, k = 20); --config picks C1..C5 (C4 and C5 are the configurations BASELINE
quotes at 2/4/8 GPUs). Between timed steps L2 is flushed by writing a 512 MB
buffer (untimed).

N > 1: one process per GPU. Launched by torchrun (RANK/WORLD_SIZE/LOCAL_RANK
in the environment) or, when --gpus N > 1 and WORLD_SIZE is unset, bench.py
re-executes itself under `python -m torch.distributed.run --nproc-per-node N
--master-addr 127.0.0.1`. Modes:
  query   (default) query sharding, target index replicated, no data-path
          collective: a self-join's ranks cluster the points identically and
          take the query clusters c with c % N == rank; a Q != T join splits
          the query rows. Strong scaling.
  target  target sharding: rank r owns T[r*nt/N, (r+1)*nt/N), joins ALL
          queries against it (partial k-lists, global indices), the partial
          lists are exchanged over NCCL (all-to-all by default) and merged
          exactly by sknn_merge_partials on the device; the step includes the
          exchange and the merge. Strong scaling.
The step time is the max over ranks of the per-rank CUDA-event time.

--impl reference: the CPU oracle (oracle/, brute force, all host cores) timed
as it stands on a bounded sample of the same workload (rank 0 only).
--launcher-selftest: exercises only the launcher / process group / max-over-
ranks reduction / JSON line (no KNN work at all; used by the CPU gloo test).
"""
from __future__ import annotations

import argparse
import json
import os
import socket
import subprocess
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
if ROOT not in sys.path:
    sys.path.insert(0, ROOT)

import datagen  # noqa: E402

PEAKS_FALLBACK = {"hbm_gbs": 6650.0, "bf16_tflops": 1590.0, "bf16_tflops_sustained": 1590.0}


def baseline_metric():
    with open(os.path.join(ROOT, "BASELINE.json")) as f:
        return json.load(f)["metric"]


def load_peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        with open(p) as f:
            d = json.load(f)
        d["_source"] = "measured (MEASURED_PEAKS.json)"
    else:
        d = dict(PEAKS_FALLBACK)
        d["sm_max_mhz"] = 1965.0
        d["_source"] = "fallback (B200_PROFILING.md)"
    # fp32 FMA pipe: measured by tools/fma_peak.cu on a B200 of this pool
    f = os.path.join(ROOT, "profiles", "r02_fma_peak.json")
    if os.path.exists(f):
        with open(f) as fh:
            m = json.load(fh)
        d["fp32_tflops"] = m["fp32_fma_tflops"]
        d["_fp32_source"] = "measured (profiles/r02_fma_peak.json, tools/fma_peak.cu)"
    else:
        d["fp32_tflops"] = 148 * 128 * 2 * d.get("sm_max_mhz", 1965.0) * 1e6 / 1e12
        d["_fp32_source"] = "derived: 148 SMs x 128 lanes x 2 flop x max SM clock"
    return d


def dist_env():
    ws = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    local = int(os.environ.get("LOCAL_RANK", "0"))
    return ws, rank, local


def free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def relaunch(ngpus):
    """--gpus N > 1 without a torchrun environment: re-execute under torchrun
    (one process per GPU, rendezvous on 127.0.0.1). Returns the exit code."""
    cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", "--nproc-per-node=%d" % ngpus,
           "--master-addr", "127.0.0.1", "--master-port", str(free_port()), os.path.abspath(__file__)] + sys.argv[1:]
    return subprocess.call(cmd)


class ClockSampler:
    """SM clock + throttle reasons sampled every 2 ms by NVML during the timed
    region (the region is milliseconds long, far below nvidia-smi's cadence);
    reports no samples when NVML is unavailable."""

    REASONS = {0x4: "sw_power_cap", 0x8: "hw_slowdown", 0x20: "sw_thermal_slowdown",
               0x40: "hw_thermal_slowdown", 0x80: "hw_power_brake_slowdown"}

    def __init__(self, device_index):
        self.dev = device_index
        self.samples, self.reasons = [], set()
        self.smax = None
        self._stop = False
        self._thr = None

    def _handle(self):
        import pynvml
        pynvml.nvmlInit()
        try:
            import torch
            p = torch.cuda.get_device_properties(self.dev)
            bus = "%08x:%02x:%02x.0" % (p.pci_domain_id, p.pci_bus_id, p.pci_device_id)
            return pynvml, pynvml.nvmlDeviceGetHandleByPciBusId(bus)
        except Exception:
            return pynvml, pynvml.nvmlDeviceGetHandleByIndex(self.dev)

    def start(self):
        import threading
        try:
            nv, h = self._handle()
            self.smax = float(nv.nvmlDeviceGetMaxClockInfo(h, nv.NVML_CLOCK_SM))
        except Exception:  # pragma: no cover - no NVML
            return

        def loop():
            while not self._stop:
                try:
                    self.samples.append(float(nv.nvmlDeviceGetClockInfo(h, nv.NVML_CLOCK_SM)))
                    bits = nv.nvmlDeviceGetCurrentClocksEventReasons(h)
                    for b, name in self.REASONS.items():
                        if bits & b:
                            self.reasons.add(name)
                except Exception:
                    pass
                time.sleep(0.002)

        self._thr = threading.Thread(target=loop, daemon=True)
        self._thr.start()

    def stop(self):
        self._stop = True
        if self._thr is not None:
            self._thr.join(timeout=2)
        return {"sm_mhz": float(np.median(self.samples)) if self.samples else None, "sm_max_mhz": self.smax,
                "samples": len(self.samples), "reasons": sorted(self.reasons), "source": "nvml, 2 ms"}


# ------------------------------------------------------------ CPU oracle --
_WORKLOADS = {}


def workload_cached(cfg_name):
    if cfg_name not in _WORKLOADS:
        _WORKLOADS[cfg_name] = datagen.workload(cfg_name)
    return _WORKLOADS[cfg_name]


def oracle_sample(cfg_name, n_queries, seed=99):
    """The oracle as it stands (brute force, fp64, all host threads) on a
    seeded sample of n_queries of the workload against ALL its targets."""
    import oracle
    Q, T, k, _ = workload_cached(cfg_name)
    rng = np.random.default_rng(seed)
    s = rng.choice(Q.shape[0], size=min(n_queries, Q.shape[0]), replace=False)
    t0 = time.perf_counter()
    oracle.knn_join(Q[s], T, k)
    return len(s), time.perf_counter() - t0, T.shape[0], k, oracle.num_threads()


def calibrate_oracle(cfg_name, target_s):
    """Number of sampled queries the oracle finishes in about target_s seconds."""
    n = 64
    while True:
        ns, dt, _, _, _ = oracle_sample(cfg_name, n, seed=98)
        if dt >= 0.5 or ns >= datagen.CONFIGS[cfg_name]["n"]:
            break
        n *= 4
    return int(max(1, min(datagen.CONFIGS[cfg_name]["n"], target_s * ns / dt)))


def cpu_baseline(cfg_name, target_s=12.0):
    n = calibrate_oracle(cfg_name, target_s)
    ns, dt, nt, k, cores = oracle_sample(cfg_name, n)
    return {"value": ns / dt, "unit": "queries/s", "cores": cores, "kind": "oracle",
            "sample": "%d seeded queries of %s against all %d targets (k=%d), %.1f s" % (ns, cfg_name, nt, k, dt)}


def run_reference(args):
    """The reference arm: the CPU oracle as it stands. Each step is a bounded
    seeded sample of the workload's queries against all targets; value =
    sampled queries / measured seconds; ms_per_step = the measured step."""
    _, rank, _ = dist_env()
    if rank != 0:
        return
    cfgd = datagen.CONFIGS[args.config]
    per_step = max(1.0, min(8.0, 120.0 / max(1, args.steps)))
    n = calibrate_oracle(args.config, per_step)
    for i in range(args.warmup):
        oracle_sample(args.config, max(1, n // 8), seed=1000 + i)
    qs, secs = 0, 0.0
    last = None
    for i in range(args.steps):
        ns, dt, nt, k, cores = oracle_sample(args.config, n, seed=2000 + i)
        qs += ns
        secs += dt
        last = (ns, dt, nt, k, cores)
    value = qs / secs
    ns, dt, nt, k, cores = last
    line = {"impl": "reference", "metric": baseline_metric(), "value": value, "unit": "queries/s",
            "n_gpus": int(args.gpus), "steps": args.steps, "warmup": args.warmup,
            "ms_per_step": 1000.0 * secs / args.steps, "higher_is_better": True, "scaling": "strong",
            "vs_baseline": None, "dtype": "f64", "data": "synthetic",
            "config": {"workload": "%s: %s" % (args.config, cfgd["desc"]), "nq": cfgd["n"], "nt": cfgd["n"],
                       "d": cfgd["d"], "k": cfgd["k"],
                       "step": "a seeded sample of %d queries against all %d targets (brute force)" % (n, nt)},
            "cpu_baseline": {"value": value, "unit": "queries/s", "cores": cores, "kind": "oracle",
                             "sample": "%d steps x %d seeded queries of %s against all %d targets (k=%d), %.1f s" % (
                                 args.steps, n, args.config, nt, k, secs)},
            "e2e": {"value": value, "unit": "queries/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


# -------------------------------------------------------------- roofline --
def roofline_of(st, stage, peaks, nq_r, nt, d, k, ws):
    """Roofline of the dominant kernel, the
    duration from CUDA events on the launching stream (stats pass).

    scan (S9-S10): bytes = query rows once + target rows as the method's reuse
    unit fetches them (rows_loaded: once per warp tile and member for the
    warp-union walk; once per query tile and member for the warp-per-query
    scan) + result rows + the bound inputs per (tile, candidate) + the center
    row per (tile, candidate that passes the bound test);
    flops = 3d per evaluated distance and per candidate-center distance +
    log2 |tc| per (query, candidate) window search. Binding = larger fraction.
    dense (S11): tensor flops = 2 KP per (query, target) pair covered by a
    dense tile and MMA term, against the dense bf16 tensor peak."""
    dpad = 4 * ((d + 3) // 4)
    out = {}
    scan_ms = stage["ms_sparse"]
    if scan_ms > 0:
        E = float(st["dist_evals_sparse"])
        C = float(st["center_evals"])
        Rl = float(st.get("rows_loaded", E))
        P = float(st["cand_pairs"]) * (nq_r / max(1.0, st["mq"] / max(1, ws)))
        tile = 32.0 if st["mapping_used"] == 1 else 8.0
        note = None
        if st["mapping_used"] != 1:
            # warp per query: rows_loaded counts every evaluation; the reuse unit of
            # §8(d) is the 8-query tile (its windows share rows through L1), so the
            # algorithmic rows are taken as rows_loaded / 8 (the tile's windows
            # coinciding: a lower bound of their union)
            Rl /= tile
            note = "warp-per-query scan: target rows counted once per 8-query tile (rows_loaded / 8)"
        # per (tile, candidate): the 16-byte cluster summary and the 4-byte center
        # distance D (every candidate is bound-tested); the center row only for
        # the candidates that pass that test (center_evals, counted per query,
        # shared by a tile's queries: C / tile)
        bytes_alg = (4.0 * dpad * nq_r + (4.0 * dpad + 4.0) * Rl + 8.0 * k * nq_r + 20.0 * P / tile +
                     4.0 * dpad * C / tile)
        flops = 3.0 * d * (E + C) + P * float(np.log2(max(2.0, nt / max(1, st["mt"]))))
        gbs = bytes_alg / (scan_ms / 1e3) / 1e9
        tfs = flops / (scan_ms / 1e3) / 1e12
        f_hbm, f_alu = gbs / peaks["hbm_gbs"], tfs / peaks["fp32_tflops"]
        if f_hbm >= f_alu:
            b = {"bound": "hbm", "achieved": gbs, "peak": peaks["hbm_gbs"], "unit": "GB/s", "frac": f_hbm}
        else:
            b = {"bound": "alu", "achieved": tfs, "peak": peaks["fp32_tflops"], "unit": "TFLOP/s", "frac": f_alu}
        if note:
            b["note"] = note
        b.update({"kernel": "k_scan_%s (level-2 scan fused with top-k)" % ("tpq" if st["mapping_used"] == 1 else "wpq"),
                  "launch_ms": scan_ms, "algorithmic_bytes": bytes_alg, "algorithmic_flops": flops,
                  "intensity_flop_per_byte": flops / bytes_alg if bytes_alg else None,
                  "hbm": {"achieved_gbs": gbs, "peak_gbs": peaks["hbm_gbs"], "frac": f_hbm},
                  "alu": {"achieved_tflops": tfs, "peak_tflops": peaks["fp32_tflops"], "frac": f_alu}})
        out["scan"] = b
    dense_ms = stage.get("ms_dense", 0.0)
    if dense_ms > 0 and st["dist_evals_dense"]:
        kp = 16 * ((dpad + 15) // 16)
        terms = float(st.get("dense_terms", 1) or 1)
        flops = 2.0 * kp * float(st["dist_evals_dense"]) * terms
        tfs = flops / (dense_ms / 1e3) / 1e12
        pk = peaks.get("bf16_tflops_sustained", peaks["bf16_tflops"])
        out["dense"] = {"bound": "tensor", "achieved": tfs, "peak": pk, "unit": "TFLOP/s", "frac": tfs / pk,
                        "kernel": "k_dense (tcgen05 bf16 dense tiles: %s)" % (
                            "exact integer, no recompute" if terms == 1 else "split-precision screen + exact recompute"),
                        "launch_ms": dense_ms, "algorithmic_flops": flops, "mma_terms": terms}
    if not out:
        return None
    dom = max(out, key=lambda s: out[s]["launch_ms"])
    r = dict(out[dom])
    r["others"] = {s: {kk: v for kk, v in out[s].items() if kk in ("kernel", "bound", "frac", "launch_ms")}
                   for s in out if s != dom}
    return r


# ------------------------------------------------------------------ main --
def launcher_selftest(args):
    """No KNN work: process group + max-over-ranks timing + the JSON line."""
    import torch
    import torch.distributed as dist
    ws, rank, _ = dist_env()
    if ws > 1:
        dist.init_process_group("gloo")
    t0 = time.perf_counter()
    time.sleep(0.01 * (rank + 1))
    ms = (time.perf_counter() - t0) * 1e3
    if ws > 1:
        t = torch.tensor([ms])
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms = float(t.item())
    if rank == 0:
        print(json.dumps({"selftest": True, "metric": baseline_metric(), "n_gpus": ws, "ms_per_step": ms,
                          "ranks_seen": ws}), flush=True)
    if ws > 1:
        dist.destroy_process_group()


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--config", default="C2")
    ap.add_argument("--mode", default="query", choices=["query", "target"])
    ap.add_argument("--exchange", default="all_to_all", choices=["all_to_all", "all_gather", "peer"])
    ap.add_argument("--global-ub", action="store_true",
                    help="target mode: prune every shard with the global level-1 bound (all-reduce MIN)")
    ap.add_argument("--shard-q-build", action="store_true",
                    help="target mode with --global-ub: the query clustering's final assignment split over the ranks")
    ap.add_argument("--prune-exchange", action="store_true",
                    help="target mode, all_to_all: send only entries at or below the min-over-ranks k-th distance")
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--mapping", default="auto")
    ap.add_argument("--launcher-selftest", action="store_true")
    args = ap.parse_args()
    args.warmup = max(args.warmup, 3)

    if args.impl == "reference":
        run_reference(args)
        return
    if args.gpus > 1 and "WORLD_SIZE" not in os.environ:
        sys.exit(relaunch(args.gpus))
    if args.launcher_selftest:
        launcher_selftest(args)
        return

    import torch
    import torch.distributed as dist

    import paper_conf_icde_chends17_b200 as sknn
    from paper_conf_icde_chends17_b200 import dist as sdist

    ws, rank, local = dist_env()
    torch.cuda.set_device(local)
    if ws > 1:
        dist.init_process_group("nccl", device_id=torch.device("cuda", local))
    dev = torch.device("cuda", local)
    stream = torch.cuda.current_stream()
    peaks = load_peaks()

    cfgd = datagen.CONFIGS[args.config]
    Qh, Th, k, self_join = workload_cached(args.config)
    nq, nt, d = Qh.shape[0], Th.shape[0], Qh.shape[1]
    Q = torch.from_numpy(Qh).to(dev)
    T = Q if self_join else torch.from_numpy(Th).to(dev)
    flush = torch.empty(512 * 1024 * 1024 // 4, dtype=torch.float32, device=dev)
    opts = dict(mapping=args.mapping)

    # ---- the per-rank step (and the stats call of its local join) ----
    if args.mode == "query":
        out_idx = torch.empty((nq, k), dtype=torch.int32, device=dev)
        out_dist = torch.empty((nq, k), dtype=torch.float32, device=dev)
        # every rank clusters all of Q identically and takes the query clusters
        # c % N == rank (dist.join_query_sharded's default partition; contiguous
        # row slices measured far worse on C4: outlier queries in a slice)
        if ws > 1:
            opts.update(shard_rank=rank, shard_count=ws)
        lo, hi = 0, nq
        Qr, Tr, oi, od = Q, (Q if self_join else T), out_idx, out_dist

        def local_join(stats=False):
            return sknn.join(Qr, Tr, k, out=(oi, od), stats=stats, stream=stream, **opts)

        def step():
            local_join()
        parallelism = "query-sharded x%d (target index replicated, no data-path collective)" % ws
        nq_rank = nq / ws
    else:
        tlo, thi = sdist.shard_bounds(nt, ws, rank)
        Tshard = T[tlo:thi].contiguous()
        group = None

        def local_join(stats=False):
            return sknn.join(Q, Tshard, min(k, thi - tlo), stats=stats, stream=stream, out_squared=1,
                             index_base=int(tlo), **opts)

        def step():
            if ws == 1 and not args.global_ub:
                local_join()
            else:
                sdist.join_target_sharded(Q, Tshard, k, tlo, group=group, exchange=args.exchange, gather=False,
                                          global_ub=args.global_ub,
                                          prune=args.prune_exchange and args.exchange == "all_to_all",
                                          **(dict(opts, shard_q_build=True) if args.shard_q_build else opts))
        parallelism = "target-sharded x%d (%s exchange of partial k-lists + exact merge%s%s)" % (
            ws, args.exchange if ws > 1 else "no", ", global level-1 bound" if args.global_ub else "",
            ", pruned by the min-over-ranks k-th" if args.prune_exchange else "")
        nq_rank = nq

    for _ in range(args.warmup):
        flush.zero_()
        step()
    torch.cuda.synchronize()

    # stats pass (untimed): per-stage CUDA events, counters and the launch
    # count of the local join; the stage split is the mean over a few joins
    stage = {"ms_build_t": 0.0, "ms_build_q": 0.0, "ms_level1": 0.0, "ms_dense": 0.0, "ms_sparse": 0.0,
             "ms_total": 0.0}
    n_stats = 3
    last = None
    for _ in range(n_stats):
        flush.zero_()
        st = local_join(stats=True)[2]
        for key in stage:
            stage[key] += st[key]
        last = st
    for key in stage:
        stage[key] /= n_stats
    launches_per_step = last["kernel_launches"] + (1 if (args.mode == "target" and ws > 1) else 0)  # + k_merge

    clocks = ClockSampler(local)
    ev = [(torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)) for _ in range(args.steps)]
    if ws > 1:
        dist.barrier()
    torch.cuda.synchronize()
    clocks.start()
    for i in range(args.steps):
        flush.zero_()                      # untimed L2 flush (512 MB > 126 MB L2)
        ev[i][0].record(stream)
        step()                             # stream-ordered, no host sync inside the join
        ev[i][1].record(stream)
    torch.cuda.synchronize()
    if ws > 1:
        dist.barrier()
    clk = clocks.stop()
    ms = [a.elapsed_time(b) for a, b in ev]
    ms_step = float(np.mean(ms))
    evals_all = float(last["dist_evals"])
    launches = launches_per_step * args.steps
    if ws > 1:
        t = torch.tensor([ms_step], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        ms_step = float(t.item())
        sums = torch.tensor([evals_all, float(launches)], dtype=torch.float64, device=dev)
        dist.all_reduce(sums)
        evals_all, launches = float(sums[0].item()), int(sums[1].item())
    value = nq / (ms_step / 1000.0)

    roof = roofline_of(last, stage, peaks, nq_rank, nt if args.mode == "query" else (thi - tlo), d, k, ws)
    if roof is not None:
        roof["peak_source"] = "HBM/bf16 %s; fp32 FMA %s" % (peaks["_source"], peaks["_fp32_source"])
        roof["share_of_step"] = roof["launch_ms"] / ms_step if ms_step else None
        roof["traffic"] = None
        tf = os.path.join(ROOT, "profiles", "traffic.json")
        if os.path.exists(tf):
            try:
                with open(tf) as f:
                    tr = json.load(f).get(args.config)
                if isinstance(tr, dict):
                    tr = tr.get(roof["kernel"].split()[0])
                roof["traffic"] = tr
            except Exception:
                pass

    # ---- end to end through the public API with host (pinned) buffers ----
    e2e = None
    if not args.no_e2e:
        e2e = measure_e2e(args, sknn, sdist, Qh, Th, k, self_join, ws, rank, dev, opts)

    cpu = None
    if rank == 0 and ws == 1 and not args.no_cpu_baseline:
        cpu = cpu_baseline(args.config)

    if rank == 0:
        pairs = float(nq) * nt
        line = {"metric": baseline_metric(), "value": value, "unit": "queries/s", "n_gpus": ws, "steps": args.steps,
                "warmup": args.warmup, "ms_per_step": ms_step, "higher_is_better": True, "scaling": "strong",
                "vs_baseline": None, "dtype": "f32", "data": "synthetic",
                "config": {"workload": "%s: %s" % (args.config, cfgd["desc"]), "nq": nq, "nt": nt, "d": d, "k": k,
                           "self_join": self_join, "mode": args.mode, "parallelism": parallelism,
                           "l2": "flushed between steps (512 MB write, untimed)", "mapping": last["mapping_used"],
                           "mq": last["mq"], "mt": last["mt"]},
                "pruned_pct": 100.0 * (1.0 - evals_all / pairs), "dist_evals": evals_all,
                "joins_per_s": 1000.0 / ms_step, "stage_ms": stage, "roofline": roof, "cpu_baseline": cpu,
                "e2e": e2e, "gpu_launches": launches, "clocks": clk}
        print(json.dumps(line), flush=True)
    if ws > 1:
        dist.barrier()
        dist.destroy_process_group()


def measure_e2e(args, sknn, sdist, Qh, Th, k, self_join, ws, rank, dev, opts):
    """The same metric through the public API with HOST buffers: every step
    copies that step's inputs from pinned host memory to the device and reads
    the step's result back (inside the timed region), then synchronises; the
    step time is the max over ranks of the host clock around it."""
    import torch
    import torch.distributed as dist
    nq, nt, d = Qh.shape[0], Th.shape[0], Qh.shape[1]
    Qp = torch.from_numpy(Qh).pin_memory()
    Tp = Qp if self_join else torch.from_numpy(Th).pin_memory()
    if args.mode == "query":
        if self_join:
            oi = torch.empty((nq, k), dtype=torch.int32).pin_memory()
            od = torch.empty((nq, k), dtype=torch.float32).pin_memory()

            def e2e_step():  # the C ABI stages the host arrays (H2D, join, D2H, sync inside)
                sknn.join(Qp, Qp, k, out=(oi, od), **opts)
            h2d, d2h = nq * d * 4, nq * k * 8
        else:  # the rank's query clusters of all of Q (opts carries shard_rank/count at N > 1)
            oi = torch.empty((nq, k), dtype=torch.int32).pin_memory()
            od = torch.empty((nq, k), dtype=torch.float32).pin_memory()

            def e2e_step():
                sknn.join(Qp, Tp, k, out=(oi, od), **opts)
            h2d, d2h = nq * d * 4 + nt * d * 4, nq * k * 8
    else:
        tlo, thi = sdist.shard_bounds(nt, ws, rank)
        Ts = Tp[tlo:thi]
        lo, hi = sdist.shard_bounds(nq, ws, rank)
        oi = torch.empty((hi - lo, k), dtype=torch.int32).pin_memory()
        od = torch.empty((hi - lo, k), dtype=torch.float32).pin_memory()
        stream = torch.cuda.current_stream()

        def e2e_step():
            dQ = Qp.to(dev, non_blocking=True)
            dT = Ts.to(dev, non_blocking=True)
            if ws == 1:
                ri, rd = sknn.join(dQ, dT, k, stream=stream, **opts)
            else:
                ri, rd = sdist.join_target_sharded(dQ, dT, k, tlo, exchange=args.exchange, gather=False,
                                                   prune=args.prune_exchange and args.exchange == "all_to_all", **opts)
            oi.copy_(ri, non_blocking=True)
            od.copy_(rd, non_blocking=True)
            torch.cuda.synchronize()
        h2d, d2h = nq * d * 4 + (thi - tlo) * d * 4, (hi - lo) * k * 8
    for _ in range(2):
        e2e_step()
    reps = max(3, args.steps // 2)
    if ws > 1:
        dist.barrier()
    t0 = time.perf_counter()
    for _ in range(reps):
        e2e_step()
    s = (time.perf_counter() - t0) / reps
    if ws > 1:
        t = torch.tensor([s], device=dev)
        dist.all_reduce(t, op=dist.ReduceOp.MAX)
        s = float(t.item())
    return {"value": nq / s, "unit": "queries/s", "h2d_bytes_per_step": int(h2d), "d2h_bytes_per_step": int(d2h),
            "ms_per_step": s * 1000.0, "per_rank_bytes": ws > 1,
            "timer": "host wall clock around the blocking call, max over ranks"}


if __name__ == "__main__":
    main()
