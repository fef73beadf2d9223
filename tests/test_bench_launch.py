"""bench.py's multi-rank launch: `python bench.py --gpus N`
with no launcher re-executes itself as N ranks through torch.distributed.run,
the children never spawn again, world == --gpus is enforced, and rank 0 prints
exactly one JSON line on stdout.  Basis: walkers are independent, so the bench
shards them one rank per GPU (§I-B, "Each thread performing the
walk is essentially executing independent of other threads").

The CPU test drives the plumbing with --launch-probe (gloo, no GPU work); the
GPU test runs the real C2 bench as 2 ranks sharing cuda:0 (gloo)."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
BENCH = os.path.join(ROOT, "bench.py")


def _env(**kw):
    env = {k: v for k, v in os.environ.items()
           if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "LOCAL_WORLD_SIZE", "MASTER_ADDR",
                        "MASTER_PORT")}
    env.update(kw)
    return env


def _json_lines(out):
    return [json.loads(ln) for ln in out.splitlines() if ln.lstrip().startswith("{")]


def test_self_launch_two_ranks_gloo():
    p = subprocess.run([sys.executable, BENCH, "--gpus", "2", "--launch-probe"],
                       env=_env(), capture_output=True, text=True, timeout=300)
    assert p.returncode == 0, p.stderr[-3000:]
    lines = _json_lines(p.stdout)
    assert len(lines) == 1, p.stdout
    # nothing but the JSON line on stdout (launcher chatter goes to stderr)
    assert len([ln for ln in p.stdout.splitlines() if ln.strip()]) == 1, p.stdout
    d = lines[0]
    assert d["n_gpus"] == 2 and d["gpus_requested"] == 2
    assert d["backend"] == "gloo"
    assert d["max_over_ranks"] == 2.0
    assert sorted(r["rank"] for r in d["per_rank"]) == [0, 1]
    assert d["feed_threads_per_rank"] == max(1, (os.cpu_count() or 1) // 2)


def test_single_rank_no_spawn():
    p = subprocess.run([sys.executable, BENCH, "--gpus", "1", "--launch-probe"],
                       env=_env(), capture_output=True, text=True, timeout=300)
    assert p.returncode == 0, p.stderr[-3000:]
    (d,) = _json_lines(p.stdout)
    assert d["n_gpus"] == 1 and d["backend"] is None


def test_world_mismatch_refused():
    # under a launcher (WORLD_SIZE set) the bench must not re-spawn, and a
    # world size different from --gpus is an error, not a silent 1-rank run
    p = subprocess.run([sys.executable, BENCH, "--gpus", "2", "--launch-probe"],
                       env=_env(WORLD_SIZE="1", RANK="0", LOCAL_RANK="0"),
                       capture_output=True, text=True, timeout=300)
    assert p.returncode != 0
    assert "--gpus 2" in p.stderr
    assert _json_lines(p.stdout) == []


@pytest.mark.gpu
def test_bench_gpus2_self_launch_on_one_gpu():
    """The driver's command shape at N = 2, both ranks on cuda:0 (gloo)."""
    p = subprocess.run([sys.executable, BENCH, "--gpus", "2", "--steps", "1", "--no-apps",
                        "--no-l1", "--no-ondemand"],
                       env=_env(GG_FORCE_DEVICE="0", GG_DIST_BACKEND="gloo"),
                       capture_output=True, text=True, timeout=1200)
    assert p.returncode == 0, p.stderr[-3000:]
    (d,) = _json_lines(p.stdout)
    assert d["n_gpus"] == 2 and d["steps"] == 1
    assert len(d["per_rank"]) == 2
    assert d["value"] > 0 and d["gpu_launches"] >= 1
    assert d["config"]["parallelism"] == "walker shards dp2, no data-path collective"
    assert len(d["e2e"]["per_rank"]) == 2
