"""bench.py's driver contract on CPU (no GPU): --gpus N self-launches N
processes under torchrun (rendezvous on 127.0.0.1) with a working process
group and max-over-ranks reduction; the reference arm prints the same metric
string as BASELINE.json and reports the time it actually ran."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _last_json(out):
    lines = [l for l in out.splitlines() if l.startswith("{")]
    assert lines, out
    return json.loads(lines[-1])


def test_bench_selflaunch_two_ranks():
    env = dict(os.environ)
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2", "--launcher-selftest"],
                       capture_output=True, text=True, timeout=300, env=env, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    line = _last_json(r.stdout)
    assert line["n_gpus"] == 2 and line["ranks_seen"] == 2
    # max over ranks: rank 1 sleeps 20 ms, rank 0 10 ms
    assert line["ms_per_step"] >= 19.0
    with open(os.path.join(ROOT, "BASELINE.json")) as f:
        assert line["metric"] == json.load(f)["metric"]


def test_reference_arm_metric_and_time():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--config", "C1",
                        "--steps", "2", "--warmup", "3"], capture_output=True, text=True, timeout=600, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    line = _last_json(r.stdout)
    with open(os.path.join(ROOT, "BASELINE.json")) as f:
        assert line["metric"] == json.load(f)["metric"]
    assert line["impl"] == "reference" and line["unit"] == "queries/s"
    # ms_per_step is the measured step (a bounded sample), consistent with value
    sample_q = int(line["config"]["step"].split()[4])
    assert abs(sample_q / (line["ms_per_step"] / 1e3) - line["value"]) / line["value"] < 0.05
    assert line["e2e"]["h2d_bytes_per_step"] == 0
