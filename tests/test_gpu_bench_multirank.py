"""bench.py's multi-rank path (torch.distributed.run, 2 ranks) on the one GPU
this environment has: both ranks share cuda:0 and use gloo collectives
(RTLSIM_BENCH_BACKEND=gloo) — the same run_sharded harness, shard offsets,
rank-0 digest gather and max-over-ranks timing the NCCL run uses. The
gathered register digests must equal a single-rank run of the same 2 x 4096
stimuli (stimuli are independent: sharding changes nothing)."""
import json
import os
import subprocess
import sys

import pytest

pytestmark = pytest.mark.gpu
ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def _bench(args, env_extra, nproc=None):
    env = dict(os.environ, **env_extra)
    if nproc:
        cmd = [sys.executable, "-m", "torch.distributed.run", "--nnodes=1", f"--nproc-per-node={nproc}",
               "--master-addr", "127.0.0.1", "--master-port", "29533", "bench.py"] + args
    else:
        cmd = [sys.executable, "bench.py"] + args
    r = subprocess.run(cmd, cwd=ROOT, env=env, capture_output=True, text=True, timeout=1500)
    assert r.returncode == 0, r.stdout[-2000:] + r.stderr[-3000:]
    lines = [l for l in r.stdout.splitlines() if l.startswith("{")]
    assert len(lines) == 1, r.stdout[-2000:]
    return json.loads(lines[0])


def test_two_rank_bench_matches_one_rank():
    common = ["--config", "3", "--steps", "3", "--warmup", "3", "--no-cpu-baseline", "--no-e2e"]
    two = _bench(["--gpus", "2", "--stimuli-per-gpu", "4096"] + common, {"RTLSIM_BENCH_BACKEND": "gloo"}, nproc=2)
    one = _bench(["--gpus", "1", "--stimuli-per-gpu", "8192"] + common, {})
    assert two["n_gpus"] == 2 and two["config"]["stimuli_total"] == 8192
    assert two["config"]["final_reg_digests_gathered"] == 8192
    assert two["config"]["final_reg_digest_xor"] == one["config"]["final_reg_digest_xor"]
    assert two["value"] > 0 and two["gpu_launches"] > 0
