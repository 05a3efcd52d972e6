"""Parity at BASELINE.json's full sizes, in the launch configuration bench.py
times (device-resident stimulus, run_device chunks): every stimulus runs on
the GPU; the oracle recomputes a deterministic sample of stimuli (tile and
shard boundaries +-1, plus seeded random ones) one by one, and the per-cycle
digest (all output words + all next-state register words), the outputs and
the final registers must be bit-identical (SURVEY §8(c) parity policy)."""
import numpy as np
import pytest

from rtlgen import shaped, stim

pytestmark = pytest.mark.gpu

FULL = {2: 4096, 3: 16384, 4: 65536}


def _sample(N, extra, seed=stim.SAMPLE_SEED):
    idx = {0, 1, 31, 32, 33, 63, 64, 127, 128, 255, 256, 1023, 1024, N // 2 - 1, N // 2, N - 2, N - 1}
    rng = np.random.default_rng(seed & 0xFFFFFFFF)
    idx |= set(int(x) for x in rng.integers(0, N, size=extra))
    return np.array(sorted(i for i in idx if 0 <= i < N))


def _run(cid, cycles, chunk, extra, s_offset=0, n=None, jit=True):
    import torch
    import oracle
    from paper_conf_icpp_linrzkh22_b200 import build, rtlsim as R
    build.build()
    ir = shaped.generate(cid)
    N = n or FULL[cid]
    seed = stim.STIM_SEED_BASE + cid
    s = torch.cuda.Stream()
    torch.cuda.set_stream(s)
    # bench.py's backend (JIT partition kernels) unless jit=False (interpreter)
    sim = R.Simulator(ir, chunk_cycles=chunk, stream=s.cuda_stream, flags=(R.F_JIT if jit else 0) | R.F_TIMING)
    d_stim = stim.stimulus_torch(ir, seed, s_offset, N, 0, cycles)
    out = torch.zeros((N, cycles, ir.OW), dtype=torch.int32, device="cuda")
    dig = torch.zeros((N, cycles), dtype=torch.int64, device="cuda")
    sim.bind_device(d_stim, N, cycles)
    # 1. the kernels bench.py times (no digest code): outputs + final registers
    sim.run_device(cycles, out)
    sim.sync()
    regs = sim.get_regs()
    pick = _sample(N, extra)
    st = stim.stimulus(ir, seed, pick + s_offset, 0, cycles)
    want = oracle.Design(ir).simulate(st, digest=True, threads=16)
    got_out = out.cpu().numpy().view(np.uint32)[pick]
    assert np.array_equal(got_out, want["out"])
    assert np.array_equal(regs[pick], want["regs"])
    # 2. check mode: per-cycle digest over every output and next-state register word
    sim.reset()
    sim.run_device(cycles, out, dig)
    sim.sync()
    got_dig = dig.cpu().numpy().view(np.uint64)[pick]
    assert np.array_equal(got_dig, want["digest"]), "per-cycle digest differs"
    assert np.array_equal(sim.get_regs()[pick], want["regs"])
    return len(pick)


def test_config2_full_size():
    assert _run(2, cycles=100, chunk=100, extra=100) > 100


def test_config3_full_size():
    assert _run(3, cycles=25, chunk=25, extra=40) > 40


def test_config3_full_size_interpreter():
    assert _run(3, cycles=12, chunk=12, extra=20, jit=False) > 20


def test_config4_full_size():
    """65536 stimuli x 25 cycles (one bench step), 24 sampled stimuli."""
    assert _run(4, cycles=25, chunk=25, extra=8) > 20


def test_config5_last_shard():
    """Config 5 (262144 stimuli over 4 GPUs): the last shard, stimuli
    196608..262143, generated from the shard offset, on this one GPU."""
    assert _run(4, cycles=4, chunk=4, extra=4, s_offset=196608, n=65536) > 16
