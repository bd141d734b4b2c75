"""bench.py's launch contract on CPU (no GPU needed): --gpus N > 1 without a launcher
re-executes itself under torch.distributed.run with N ranks (rank 0 prints ONE line with
n_gpus = N, the other ranks exit 0), and a world size that differs from --gpus is refused.
The reference arm (O3 on the host) is what runs here; the GPU arm needs a B200."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def run(args, env=None):
    e = dict(os.environ)
    e.pop("WORLD_SIZE", None)
    e.update(env or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True, text=True,
                          timeout=600, env=e, cwd=ROOT)


def test_two_rank_spawn_prints_one_line():
    p = run(["--gpus", "2", "--impl", "reference", "--config", "c1", "--steps", "2", "--warmup", "1"])
    assert p.returncode == 0, p.stderr[-2000:]
    lines = [json.loads(x) for x in p.stdout.splitlines() if x.startswith("{")]
    assert len(lines) == 1
    assert lines[0]["n_gpus"] == 2 and lines[0]["impl"] == "reference" and lines[0]["value"] > 0
    assert lines[0]["cpu_baseline"]["kind"] == "oracle" and lines[0]["e2e"]["h2d_bytes_per_step"] == 0


def test_world_size_must_match_gpus():
    p = run(["--gpus", "4", "--impl", "reference", "--config", "c1"], env={"WORLD_SIZE": "2"})
    assert p.returncode != 0 and "WORLD_SIZE" in (p.stderr + p.stdout)
