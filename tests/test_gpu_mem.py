"""Memories on the GPU (ARRSEL reads + synchronous write ports; PAPER.md
§3.1.1 Fig 5, reading 12) against the CPU oracle, bit for bit:
every output, every register, every per-cycle digest and the final memory
contents, on the closed-form pin designs and register-file designs (wide
three-word entries, 1-bit entries, out-of-range addresses, two partitions)."""
import numpy as np
import pytest

from rtlgen import designs, stim

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def R():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_icpp_linrzkh22_b200 import build, rtlsim
    build.build()
    return rtlsim


def _check(R, oracle_lib, ir, st, chunk=16, **opt):
    want = oracle_lib.Design(ir).simulate(st, digest=True, mems=True, threads=8)
    sim = R.Simulator(ir, chunk_cycles=chunk, flags=R.F_JIT | opt.pop("flags", 0), **opt)
    sim.bind(st)
    got = sim.run(st.shape[1], out=True, regs=True, digest=True)
    assert np.array_equal(got["out"], want["out"]), "outputs"
    assert np.array_equal(got["regs"], want["regs"]), "registers"
    assert np.array_equal(got["digest"], want["digest"]), "digest"
    assert np.array_equal(sim.get_mems(), want["mems"]), "memory contents"
    return sim


def test_memseq(R, oracle_lib):
    ir = designs.mem_seq_dut()
    _check(R, oracle_lib, ir, np.zeros((70, 300, 0), np.uint32), chunk=37)


def test_mem_bounds_random(R, oracle_lib):
    ir = designs.mem_bounds_dut()
    st = stim.stimulus(ir, 0xB0B, np.arange(100), 0, 64)
    _check(R, oracle_lib, ir, st)


def test_mem_two_ports(R, oracle_lib):
    _check(R, oracle_lib, designs.mem_two_port_dut(), np.zeros((33, 40, 0), np.uint32), chunk=8)


@pytest.mark.parametrize("seed,parts,lanes", [(1, 1, 0), (2, 2, 0), (3, 1, 1), (4, 2, 4)])
def test_regfile(R, oracle_lib, seed, parts, lanes):
    ir = designs.regfile_dut(seed=seed, depth=32, width=32, n_read=3, parts=parts)
    st = stim.stimulus(ir, 0x5EED + seed, np.arange(130), 0, 50)
    sim = _check(R, oracle_lib, ir, st, op_lanes=lanes)
    # reset: memories return to their initial contents
    sim.reset()
    got = sim.run(10, out=True, regs=False)
    want = oracle_lib.Design(ir).simulate(st[:, :10], digest=False, mems=True)
    assert np.array_equal(got["out"], want["out"]) and np.array_equal(sim.get_mems(), want["mems"])


def test_regfile_generic_addressing(R, oracle_lib, monkeypatch):
    monkeypatch.setenv("RTLSIM_JIT_GENERIC", "1")
    ir = designs.regfile_dut(seed=9, depth=16, width=40, n_read=2)
    _check(R, oracle_lib, ir, stim.stimulus(ir, 0x99, np.arange(45), 0, 30))


def test_memories_need_jit(R):
    with pytest.raises(R.RtlsimError) as ei:
        R.Simulator(designs.mem_seq_dut())
    assert ei.value.code == -4
