"""Multi-process host logic of the stimulus-sharding harness on CPU (gloo,
world_size 2): shard math, elapsed-time max-reduction and digest/register
gathers reproduce the single-process result. The oracle stands in for the
GPU compute step (this test never touches the CUDA path)."""
import os
import socket
import sys

import numpy as np
import pytest

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_shard_range_partitions():
    from paper_conf_icpp_linrzkh22_b200.parallel import shard_range
    for n_total in (0, 1, 7, 64, 1000, 262144):
        for world in (1, 2, 3, 4, 8):
            covered = []
            for r in range(world):
                s0, n = shard_range(n_total, world, r)
                covered.extend(range(s0, s0 + n))
            assert covered == list(range(n_total))
    assert shard_range(262144, 4, 1) == (65536, 65536)    # config 5 at 4 GPUs = config 4 per GPU


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def _worker(rank, world, port, n_total, T, q):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch.distributed as dist
    import oracle
    from rtlgen import designs, stim
    from paper_conf_icpp_linrzkh22_b200.parallel import run_sharded
    dist.init_process_group("gloo", rank=rank, world_size=world)
    ir = designs.tiny_dut()
    d = oracle.Design(ir)

    def simulate(s0, n):
        st = stim.tiny_stimulus(99, np.arange(s0, s0 + n), T)
        r = d.simulate(st, digest=True)
        return {"digest": r["digest"], "regs": r["regs"], "elapsed": 0.1 * (rank + 1)}

    res = run_sharded(simulate, n_total)
    if rank == 0:
        q.put((res.elapsed_max, res.digest, res.regs))
    dist.destroy_process_group()


def test_two_rank_gather_matches_single_process(oracle_lib):
    import multiprocessing as mp
    from rtlgen import designs, stim
    n_total, T, world = 37, 12, 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, n_total, T, q)) for r in range(world)]
    for p in ps:
        p.start()
    el, dig, regs = q.get(timeout=180)
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    ir = designs.tiny_dut()
    want = oracle_lib.simulate(ir, stim.tiny_stimulus(99, np.arange(n_total), T), digest=True)
    assert el == pytest.approx(0.2)                      # max over ranks
    assert np.array_equal(dig, want["digest"]) and np.array_equal(regs, want["regs"])
