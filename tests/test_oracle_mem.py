"""Pins of the oracle's memories (ARRSEL read op MEMRD + synchronous write
ports; §3.1.1 Fig 5, reading 12) by closed forms — a
counter-driven memory whose contents at every cycle follow from the counter,
read-during-write returning the pre-edge value, out-of-range reads giving 0
and out-of-range writes changing nothing, the later of two ports winning —
and by brute force against the pure-Python loop (oracle.pysim) on a
register-file design with wide and 1-bit memories."""
import numpy as np
import pytest

from rtlgen import designs, stim
from rtlgen import ir as I


def test_memseq_closed_form(oracle_lib):
    ir = designs.mem_seq_dut()
    T = 300
    r = oracle_lib.simulate(ir, np.zeros((2, T, 0), np.uint32), mems=True)
    out = r["out"][0]
    c = np.arange(T) % 256
    assert np.array_equal(out[:, 0], c)                          # the counter
    want_prev = np.where(np.arange(T) >= 1, c, designs.MEMSEQ_INIT[7])
    assert np.array_equal(out[:, 1], want_prev)                  # written last cycle
    want_same = np.where(np.arange(T) >= 8, (np.arange(T) - 7) % 256,
                         np.asarray(designs.MEMSEQ_INIT)[np.arange(T) % 8])
    assert np.array_equal(out[:, 2], want_same)                  # read-during-write: old value
    # final memory: entry e holds the last value written there, (k + 1) mod 256
    # for the last cycle k < T with k mod 8 == e
    last = [max(k for k in range(T) if k % 8 == e) for e in range(8)]
    assert r["mems"][0].tolist() == [(k + 1) % 256 for k in last]
    assert np.array_equal(r["mems"][0], r["mems"][1])


def test_mem_bounds(oracle_lib):
    ir = designs.mem_bounds_dut()
    rng = np.random.default_rng(3)
    N, T = 16, 40
    st = np.zeros((N, T, 4), np.uint32)
    st[:, :, 0] = 1                                              # we
    st[:, :, 1] = rng.integers(5, 8, size=(N, T))                # waddr: never a real entry
    st[:, :, 2] = rng.integers(0, 1 << 16, size=(N, T))
    st[:, :, 3] = rng.integers(0, 8, size=(N, T))                # raddr: any
    r = oracle_lib.simulate(ir, st, mems=True)
    init = np.asarray(designs.MEMB_INIT + [0, 0, 0])
    assert np.array_equal(r["out"][:, :, 0], init[st[:, :, 3]])  # out of range reads 0
    assert np.array_equal(r["mems"], np.tile(designs.MEMB_INIT, (N, 1)))   # nothing written
    # one in-range write of 0xBEEF to entry 2 at cycle 5: visible from cycle 6
    st[:, 5, 1], st[:, 5, 2] = 2, 0xBEEF
    st[:, :, 3] = 2
    r = oracle_lib.simulate(ir, st, mems=True)
    assert np.all(r["out"][:, :6, 0] == designs.MEMB_INIT[2]) and np.all(r["out"][:, 6:, 0] == 0xBEEF)
    # the enable: the same write with we = 0 changes nothing
    st[:, 5, 0] = 0
    r = oracle_lib.simulate(ir, st, mems=True)
    assert np.all(r["out"][:, :, 0] == designs.MEMB_INIT[2])


def test_mem_later_port_wins(oracle_lib):
    ir = designs.mem_two_port_dut()
    T = 50
    r = oracle_lib.simulate(ir, np.zeros((1, T, 0), np.uint32))
    out = r["out"][0]
    c = np.arange(T)
    assert np.array_equal(out[1:, 1], (~(c[1:] - 1)) & 0xFF)
    assert out[0, 1] == 0                                        # entry 3 not yet written


@pytest.mark.parametrize("seed", [1, 2])
def test_regfile_vs_pysim(oracle_lib, seed):
    from oracle import pysim
    ir = designs.regfile_dut(seed=seed, depth=16, width=40, n_read=3)
    st = stim.stimulus(ir, 0x77 + seed, np.arange(6), 0, 30)
    got = oracle_lib.simulate(ir, st, mems=True)
    out, regs, mems = pysim.simulate(ir, st)
    assert np.array_equal(got["out"], out) and np.array_equal(got["regs"], regs)
    assert np.array_equal(got["mems"], mems)


def test_mem_validation(oracle_lib):
    ir = designs.mem_seq_dut()
    ir.ops["imm"][ir.ops["opcode"] == I.OPCODES["MEMRD"]] = 5        # no such memory
    with pytest.raises(ValueError):
        oracle_lib.Design(ir)
