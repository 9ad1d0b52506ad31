"""CPU check of bench.py's multi-rank plumbing (VERDICT r1 'multi-GPU readiness'):
`python bench.py --gpus 2 --dry-run` with no torchrun environment must start 2 ranks itself
(torch.distributed.run, 127.0.0.1), shard reference ids into contiguous ranges covering
[0, R_total), merge the per-rank top-k in the shared total order over the process group
(gloo here, NCCL on GPUs) and have rank 0 alone print one JSON line.  No matching runs (no CPU
stand-in for the product path): each rank ranks synthetic counts, and the merge must equal the
global ranking with every planted target first."""
import json
import os
import subprocess
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _run(n):
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    p = subprocess.run([sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", str(n), "--dry-run"],
                       capture_output=True, text=True, timeout=300, env=env, cwd=ROOT)
    assert p.returncode == 0, p.stderr[-3000:]
    lines = [l for l in p.stdout.splitlines() if l.strip()]
    assert len(lines) == 1, p.stdout  # rank 0 only, one line
    return json.loads(lines[0])


def test_bench_self_launches_two_ranks():
    out = _run(2)
    assert out["dry_run"] and out["n_gpus"] == 2
    spans = [tuple(s) for s in out["shards"]]
    assert spans[0][0] == 0 and spans[-1][1] == out["refs_total"]
    assert all(spans[i][1] == spans[i + 1][0] for i in range(len(spans) - 1))
    assert out["planted_top1"] == 1.0 and out["merge_equals_global"]


def test_bench_dry_run_single_rank():
    out = _run(1)
    assert out["n_gpus"] == 1 and [tuple(s) for s in out["shards"]] == [(0, out["refs_total"])]
    assert out["planted_top1"] == 1.0
