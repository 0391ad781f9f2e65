"""bench.py's N-rank plumbing on CPU: `--gpus N` launches N ranks itself (torch.distributed.run
on 127.0.0.1, gloo under --dry-run), every rank builds its share of every logical problem
with dist.partition, and rank 0 prints ONE line whose n_gpus is N and whose shares tile
each problem exactly once (SURVEY 8(d) configs[1,3,4] at N > 1, 8(e))."""
import json
import os
import subprocess
import sys

import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(*args):
    env = dict(os.environ)
    for k in ("WORLD_SIZE", "RANK", "LOCAL_RANK", "MASTER_ADDR", "MASTER_PORT"):
        env.pop(k, None)
    r = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), *args], capture_output=True,
                       text=True, timeout=240, env=env, cwd=ROOT)
    assert r.returncode == 0, r.stderr[-2000:]
    lines = [ln for ln in r.stdout.splitlines() if ln.startswith("{")]
    assert len(lines) == 1, r.stdout
    return json.loads(lines[0])


@pytest.mark.parametrize("gpus,workload,rows,splitk", [
    (2, "sweep", 26, 16),       # R >= 2*1024: 2^11..2^23 rows x 2 layouts = 26; the rest split-K
    (4, "rowshard", 1, 0),      # configs[3]: 131072 rows -> row blocks, no collective
    (2, "splitk", 0, 1),        # configs[4]: 1024 outputs -> split-K + all_reduce
])
def test_bench_self_launches_n_ranks(gpus, workload, rows, splitk):
    line = _run("--gpus", str(gpus), "--dry-run", "--workload", workload)
    assert line["n_gpus"] == gpus
    assert line["dry_run"] and line["shares_tile_problems"]
    assert line["scaling"] == "strong"
    assert line["config"]["shares"] == {"rows": rows, "splitk": splitk}
    assert line["max_rank_probe"] == gpus - 1          # max over ranks of each rank's id


def test_bench_single_rank_dry_run():
    line = _run("--dry-run")
    assert line["n_gpus"] == 1 and line["shares_tile_problems"]
    assert line["config"]["shares"] == {"rows": 42, "splitk": 0}
