"""Multi-process host logic of the stimulus-sharding harness on CPU (gloo,
world_size 2) — exactly the code bench.py runs under NCCL
(paper_conf_icpp_linrzkh22_b200.parallel.run_sharded), with the oracle
standing in for the GPU compute step (this test never touches the CUDA
path): shard math, the elapsed-time MAX reduction, the rank-0 gather of
per-stimulus register digests and the all_gather + OR of toggle coverage
reproduce the single-process result."""
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
    # config 5: 262144 stimuli over 2 / 4 / 8 GPUs
    assert shard_range(262144, 2, 1) == (131072, 131072)
    assert shard_range(262144, 4, 3) == (196608, 65536)
    assert shard_range(262144, 8, 5) == (163840, 32768)


def _free_port():
    s = socket.socket()
    s.bind(("127.0.0.1", 0))
    p = s.getsockname()[1]
    s.close()
    return p


def reg_digest_ref(regs):
    from rtlgen.stim import _mix_np
    k = np.arange(regs.shape[1], dtype=np.uint64)
    z = ((k + np.uint64(1 + 0x80000000)) << np.uint64(32)) | regs.astype(np.uint64)
    with np.errstate(over="ignore"):
        return np.bitwise_xor.reduce(_mix_np(z), axis=1)


def oracle_shard(ir, s0, n, T):
    """Oracle stand-in for one shard: final register digests + coverage."""
    import oracle
    from rtlgen import stim
    d = oracle.Design(ir)
    st = stim.tiny_stimulus(99, np.arange(s0, s0 + n), T)
    r = np.tile(np.asarray(ir.reg_init, np.uint32), (n, 1))
    cov = np.zeros(ir.RW, np.uint32)
    for c in range(T if n else 0):
        r2 = d.simulate(st[:, c:c + 1], regs_in=r, out=False, regs=True)["regs"]
        if n:
            cov |= np.bitwise_or.reduce(r ^ r2, axis=0)
        r = r2
    return reg_digest_ref(r) if n else np.zeros(0, np.uint64), cov


def _worker(rank, world, port, n_total, T, q):
    sys.path.insert(0, ROOT)
    os.environ.update(MASTER_ADDR="127.0.0.1", MASTER_PORT=str(port))
    import torch.distributed as dist
    from rtlgen import designs
    from paper_conf_icpp_linrzkh22_b200.parallel import run_sharded
    dist.init_process_group("gloo", rank=rank, world_size=world)
    ir = designs.tiny_dut()

    def simulate(s0, n):
        dg, cov = oracle_shard(ir, s0, n, T)
        return {"reg_digest": dg, "coverage": cov, "elapsed": 0.1 * (rank + 1), "s0": s0, "n": n}

    res = run_sharded(simulate, n_total)
    q.put((rank, res.elapsed_max, res.reg_digest, res.coverage, res.local["s0"], res.local["n"]))
    dist.destroy_process_group()


@pytest.mark.parametrize("n_total", [37, 1])
def test_two_rank_gather_matches_single_process(oracle_lib, n_total):
    import multiprocessing as mp
    from rtlgen import designs
    T, world = 12, 2
    ctx = mp.get_context("spawn")
    q = ctx.Queue()
    port = _free_port()
    ps = [ctx.Process(target=_worker, args=(r, world, port, n_total, T, q)) for r in range(world)]
    for p in ps:
        p.start()
    got = sorted([q.get(timeout=180) for _ in range(world)], key=lambda x: x[0])
    for p in ps:
        p.join(timeout=60)
        assert p.exitcode == 0
    ir = designs.tiny_dut()
    want_dig, want_cov = oracle_shard(ir, 0, n_total, T)
    for rank, el, dig, cov, s0, n in got:
        assert el == pytest.approx(0.2)                      # max over ranks
        assert np.array_equal(cov, want_cov)                 # OR over ranks, on every rank
        if rank == 0:
            assert dig.dtype == np.uint64 and np.array_equal(dig, want_dig)
        else:
            assert dig is None                               # gathered to rank 0 only
    assert [(s0, n) for _, _, _, _, s0, n in got] == [(0, (n_total + 1) // 2), ((n_total + 1) // 2, n_total // 2)]
