"""bench.py's launch contract on CPU: `--gpus N` outside torchrun re-launches itself under torch.distributed.run with
N ranks (127.0.0.1 rendezvous); the reference arm (the fp64 oracle) prints ONE JSON line from rank 0 carrying n_gpus
= N, scaling "weak", the product arm's config object and the cpu_baseline / e2e keys."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _json_lines(out):
    return [json.loads(ln) for ln in out.splitlines() if ln.startswith("{")]


def test_bench_gpus2_spawns_two_ranks_reference_arm():
    env = dict(os.environ)
    env.pop("WORLD_SIZE", None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--gpus", "2",
                        "--steps", "1", "--warmup", "3", "--ref-band", "8"], cwd=ROOT, env=env,
                       capture_output=True, text=True, timeout=600)
    assert r.returncode == 0, r.stderr[-3000:]
    lines = _json_lines(r.stdout)
    assert len(lines) == 1, r.stdout[-2000:]
    ln = lines[0]
    assert ln["impl"] == "reference" and ln["n_gpus"] == 2 and ln["scaling"] == "weak"
    assert ln["unit"] == "frames/s" and ln["value"] > 0 and ln["steps"] == 1 and ln["warmup"] == 3
    assert ln["config"]["frames_per_rank"] == 30 and "DP training" in ln["config"]["parallelism"]
    assert ln["cpu_baseline"]["kind"] == "oracle" and ln["cpu_baseline"]["cores"] >= 1
    assert ln["e2e"]["h2d_bytes_per_step"] == 0


def test_bench_rejects_too_few_warmup_steps():
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--impl", "reference", "--warmup", "1"],
                       cwd=ROOT, capture_output=True, text=True, timeout=120)
    assert r.returncode != 0
