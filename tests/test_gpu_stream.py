"""The streaming boundary (rtlsim_bind_stream / rtlsim_run_stream): the
producer / consumer ends of the paper's stimulus-group pipeline (PAPER.md
§3.2.3, Fig 11), checked bit for bit against the CPU oracle:
several chunks with a ragged last one, ragged N, digest on and off, cursor
continuation across calls, and the producer / consumer abort paths."""
import numpy as np
import pytest

from rtlgen import designs, shaped, stim
from paper_conf_icpp_linrzkh22_b200 import rtlsim as Rmod

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def R():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_icpp_linrzkh22_b200 import build
    build.build()
    return Rmod


def _design(kind):
    if kind == "tiny":
        ir = designs.tiny_dut()
        return ir, lambda idx, T: stim.tiny_stimulus(stim.STIM_SEED_BASE + 1, idx, T, mode="B")
    ir = shaped.generate(3, scale=0.05)
    return ir, lambda idx, T: stim.stimulus(ir, 0xABCD, idx, 0, T)


def _collect(N, T, OW):
    got = {"out": np.zeros((N, T, OW), np.uint32), "digest": np.zeros((N, T), np.uint64), "calls": []}

    def consume(c0, out, dig):
        nc = out.shape[1]
        got["calls"].append((c0, nc, dig is not None))
        got["out"][:, c0:c0 + nc] = out
        if dig is not None:
            got["digest"][:, c0:c0 + nc] = dig
        return True
    return got, consume


@pytest.mark.parametrize("kind,N,T,chunk,flags", [
    ("tiny", 100, 37, 8, 0),                     # 5 chunks, last one 5 cycles, ragged N
    ("tiny", 64, 20, 7, Rmod.F_DIGEST),          # digest on, chunk not dividing T
    ("shaped", 45, 23, 6, Rmod.F_DIGEST | Rmod.F_JIT),
    ("shaped", 33, 16, 16, 0),                   # one chunk
])
def test_stream_bind_and_run(R, oracle_lib, kind, N, T, chunk, flags):
    ir, gen = _design(kind)
    st = gen(np.arange(N), T)
    want = oracle_lib.simulate(ir, st, digest=True, threads=8)
    sim = R.Simulator(ir, chunk_cycles=chunk, flags=flags)
    produced = []

    def produce(c0, nc):
        produced.append((c0, nc))
        return st[:, c0:c0 + nc]

    sim.bind_stream(N, T, produce)
    got, consume = _collect(N, T, sim.OW)
    # two calls: the cycle cursor continues across them
    t1 = T // 3
    sim.run_stream(t1, consume)
    sim.run_stream(T - t1, consume)
    assert np.array_equal(got["out"], want["out"])
    assert np.array_equal(sim.get_regs(), want["regs"])
    dig_on = bool(flags & Rmod.F_DIGEST)
    assert all(d == dig_on for _, _, d in got["calls"])
    if dig_on:
        assert np.array_equal(got["digest"], want["digest"])
    # chunks arrive in cycle order and tile [0, T) exactly, on both ends
    for calls in (produced, [(c, n) for c, n, _ in got["calls"]]):
        assert [c for c, _ in calls] == sorted(c for c, _ in calls)
        assert sum(n for _, n in calls) == T and all(1 <= n <= chunk for _, n in calls)


def test_run_stream_after_host_bind(R, oracle_lib):
    ir, gen = _design("tiny")
    st = gen(np.arange(70), 30)
    want = oracle_lib.simulate(ir, st, digest=True)
    sim = R.Simulator(ir, chunk_cycles=9, flags=Rmod.F_DIGEST)
    sim.bind(st)
    got, consume = _collect(70, 30, sim.OW)
    sim.run_stream(30, consume)
    assert np.array_equal(got["out"], want["out"]) and np.array_equal(got["digest"], want["digest"])


def test_producer_abort(R, oracle_lib):
    ir, gen = _design("tiny")
    N, T, chunk = 40, 40, 8
    st = gen(np.arange(N), T)
    want = oracle_lib.simulate(ir, st, digest=False)
    sim = R.Simulator(ir, chunk_cycles=chunk)
    sim.bind_stream(N, T, lambda c0, nc: None if c0 >= 16 else st[:, c0:c0 + nc])
    got, consume = _collect(N, T, sim.OW)
    with pytest.raises(Rmod.RtlsimError) as ei:
        sim.run_stream(T, consume)
    assert ei.value.code == -1 and "producer aborted" in str(ei.value)
    # cycles 0..15 were simulated (two chunks): registers are the oracle's after 16 cycles
    want16 = oracle_lib.simulate(ir, st[:, :16], digest=False)
    assert np.array_equal(sim.get_regs(), want16["regs"])
    assert np.array_equal(got["out"][:, :8], want["out"][:, :8])
    # the ctx is not sticky-failed: reset and a full run from a working producer
    sim.bind_stream(N, T, lambda c0, nc: st[:, c0:c0 + nc])
    got2, consume2 = _collect(N, T, sim.OW)
    sim.run_stream(T, consume2)
    assert np.array_equal(got2["out"], want["out"]) and np.array_equal(sim.get_regs(), want["regs"])


def test_consumer_abort(R, oracle_lib):
    ir, gen = _design("tiny")
    N, T, chunk = 40, 40, 8
    st = gen(np.arange(N), T)
    want = oracle_lib.simulate(ir, st, digest=True)
    sim = R.Simulator(ir, chunk_cycles=chunk, flags=Rmod.F_DIGEST)
    sim.bind(st)
    seen = []

    def consume(c0, out, dig):
        seen.append(c0)
        return c0 < 8          # refuse the second chunk
    with pytest.raises(Rmod.RtlsimError) as ei:
        sim.run_stream(T, consume)
    assert ei.value.code == -1 and "consumer aborted" in str(ei.value)
    assert seen == [0, 8]
    # the refused chunk (8..15) and at most the one launched after it were simulated
    regs = sim.get_regs()
    ok = [c for c in (16, 24) if np.array_equal(regs, oracle_lib.simulate(ir, st[:, :c])["regs"])]
    assert ok, "register state is not at a chunk boundary after the abort"
    sim.reset()
    got, consume2 = _collect(N, T, sim.OW)
    sim.run_stream(T, consume2)
    assert np.array_equal(got["out"], want["out"]) and np.array_equal(got["digest"], want["digest"])
