"""bench.py's multi-GPU launcher on CPU: `--gpus 2` outside torchrun re-launches itself as two ranks
(torch.distributed.run on 127.0.0.1) that join a gloo process group; rank 0 prints the one JSON line
with n_gpus = 2 (the reference arm is CPU code, so it runs here)."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env_extra=None):
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    env.update(env_extra or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True,
                          text=True, timeout=600, env=env, cwd=ROOT)


def test_launcher_world2_gloo():
    r = _run(["--impl", "reference", "--gpus", "2", "--config", "C1", "--steps", "1", "--warmup", "3",
              "--ref-seconds", "1"])
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [json.loads(s) for s in r.stdout.splitlines() if s.startswith("{")]
    assert len(lines) == 1, r.stdout  # rank 0 alone prints
    line = lines[0]
    assert line["impl"] == "reference" and line["n_gpus"] == 2 and line["ranks"] == 2
    assert line["value"] > 0 and line["e2e"]["value"] == line["value"]


def test_world_size_must_match_gpus():
    r = _run(["--impl", "reference", "--gpus", "4", "--config", "C1", "--steps", "1"],
             {"WORLD_SIZE": "2", "RANK": "0", "LOCAL_RANK": "0"})
    assert r.returncode == 2 and "WORLD_SIZE=2" in r.stderr
