"""bench.py --gpus N starts N ranks itself (one process per GPU via
torch.distributed.run on 127.0.0.1) when it is not already under torchrun, and
refuses a WORLD_SIZE that differs from --gpus: a SCALE run can never silently
measure one rank.  Checked on CPU with the gloo backend."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(args, env=None):
    e = dict(os.environ)
    for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT"):
        e.pop(k, None)
    e.update(env or {})
    return subprocess.run([sys.executable, os.path.join(ROOT, "bench.py")] + args, capture_output=True, text=True,
                          timeout=300, env=e, cwd=ROOT)


def test_bench_spawns_ranks():
    r = _run(["--gpus", "2", "--launcher-check"])
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [json.loads(x) for x in r.stdout.splitlines() if x.startswith("{")]
    assert len(lines) == 1, r.stdout                     # rank 0 only
    assert lines[0]["n_gpus"] == 2 and lines[0]["ranks"] == 2
    assert lines[0]["ms_max"] == 2.0                     # max over ranks (rank r reports r+1)


def test_bench_rejects_world_mismatch():
    r = _run(["--gpus", "2", "--launcher-check"], env={"WORLD_SIZE": "1", "RANK": "0", "LOCAL_RANK": "0"})
    assert r.returncode == 2
    assert "WORLD_SIZE=1 but --gpus 2" in r.stderr
