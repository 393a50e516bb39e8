"""The multi-rank path of bench.py (self-launch of N ranks, seed sharding, barriers,
max-over-ranks timing, the map reduce through sharding.reduce_map, the JSON line) run end to
end on ONE GPU: both ranks use cuda:0 and the gloo backend (NCCL cannot put two ranks on one
device).  The reduced map rank 0 ends with must equal the oracle's map of the whole
workload bit for bit.  On an 8-GPU box the same code runs with NCCL, one rank per GPU."""
from __future__ import annotations

import json
import os
import subprocess
import sys

import numpy as np
import pytest

import oracle
import phantom

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.mark.gpu
@pytest.mark.parametrize("world", [2, 3])
def test_bench_ranks_one_gpu_map_equals_oracle(world, tmp_path):
    import torch
    if not torch.cuda.is_available():
        pytest.skip("needs a CUDA device")
    env = {k: v for k, v in os.environ.items() if k not in ("WORLD_SIZE", "RANK", "LOCAL_RANK")}
    env.update(BENCH_DIST_BACKEND="gloo", BENCH_SINGLE_DEVICE="1")
    dump = str(tmp_path / "map.npy")
    cmd = [sys.executable, os.path.join(ROOT, "bench.py"), "--gpus", str(world), "--steps", "2", "--warmup", "3",
           "--config", "c2_dispersed", "--no-cpu-baseline", "--no-gather-bench", "--no-lengths",
           "--dump-map", dump]
    out = subprocess.run(cmd, capture_output=True, text=True, timeout=1200, cwd=ROOT, env=env)
    assert out.returncode == 0, out.stderr[-3000:]
    lines = [l for l in out.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, out.stdout
    d = json.loads(lines[0])
    assert d["n_gpus"] == world and d["value"] > 0 and d["config"]["seeds"] == 1000
    assert d["config"]["parallelism"].startswith(f"seed-sharded x{world}")
    for r in range(world):
        assert f"[bench rank {r}/{world}]" in out.stderr
    gm = np.load(dump)
    w = phantom.config("c2_dispersed")
    ref = oracle.track(w, want_particles=False, threads=max(1, len(os.sched_getaffinity(0))))["map"]
    assert np.array_equal(gm.astype(np.uint64), ref)
    assert int(ref.sum()) == d["config"]["steps_per_pass"]
