"""Brute force and invariants for the oracle on random DAGs — CPU only.

* exhaustive truth tables of random combinational DAGs (<= 16 input bits,
  all opcodes, widths across every word boundary) against the pure-Python
  big-int evaluator (oracle/pysim.py),
* sequential random designs over several cycles against pysim,
* invariants that hold for any correct simulator: stimulus permutation,
  run splitting through regs_in, single vs multi-threaded, digest recomputed
  from the outputs and final registers.
"""
import numpy as np
import pytest

from rtlgen import designs, stim
from oracle import pysim


@pytest.mark.parametrize("seed", range(6))
def test_comb_dag_exhaustive(oracle_lib, seed):
    ir = designs.random_dag(seed, n_ops=60 + 25 * seed, input_widths=(3, 5, 1, 4, 3))
    st = designs.exhaustive_stimulus(ir)          # 2^16 stimuli, 1 cycle
    got = oracle_lib.simulate(ir, st)["out"]
    idx = np.random.default_rng(seed).choice(st.shape[0], 384, replace=False)
    idx = np.concatenate([idx, [0, 1, st.shape[0] - 1]])
    want, _ = pysim.simulate(ir, st[idx])
    assert np.array_equal(got[idx], want)


@pytest.mark.parametrize("seed", range(4))
def test_comb_dag_tiny_inputs_full_table(oracle_lib, seed):
    """<= 9 input bits: the whole truth table through pysim."""
    ir = designs.random_dag(100 + seed, n_ops=40, input_widths=(4, 3, 2))
    st = designs.exhaustive_stimulus(ir)
    got = oracle_lib.simulate(ir, st)["out"]
    want, _ = pysim.simulate(ir, st)
    assert np.array_equal(got, want)


@pytest.mark.parametrize("seed", range(4))
def test_sequential_dag_vs_pysim(oracle_lib, seed):
    ir = designs.random_dag(200 + seed, n_ops=80, n_regs=10, input_widths=(7, 33, 1, 64))
    st = stim.stimulus(ir, 0x1234 + seed, np.arange(12), 0, 9)
    r = oracle_lib.simulate(ir, st)
    want_o, want_r = pysim.simulate(ir, st)
    assert np.array_equal(r["out"], want_o)
    assert np.array_equal(r["regs"], want_r)


def test_invariants(oracle_lib):
    ir = designs.random_dag(300, n_ops=120, n_regs=12, input_widths=(9, 40, 1, 5))
    N, T = 40, 30
    st = stim.stimulus(ir, 77, np.arange(N), 0, T)
    d = oracle_lib.Design(ir)
    full = d.simulate(st, digest=True)
    # permutation of stimuli permutes results
    perm = np.random.default_rng(1).permutation(N)
    p = d.simulate(st[perm], digest=True)
    assert np.array_equal(p["out"], full["out"][perm]) and np.array_equal(p["regs"], full["regs"][perm])
    # run splitting: T1 then T2 from the saved registers
    a = d.simulate(st[:, :13])
    b = d.simulate(st[:, 13:], regs_in=a["regs"])
    assert np.array_equal(np.concatenate([a["out"], b["out"]], axis=1), full["out"])
    assert np.array_equal(b["regs"], full["regs"])
    # threads
    m = d.simulate(st, digest=True, threads=5)
    for k in ("out", "regs", "digest"):
        assert np.array_equal(m[k], full[k])


def test_digest_definition(oracle_lib):
    """digest[s][c] = XOR_j mix((j+1)<<32 | O_c[j]) ^ XOR_k mix((k+1+2^31)<<32 | R_{c+1}[k])."""
    ir = designs.random_dag(400, n_ops=50, n_regs=6, input_widths=(8, 8))
    N, T = 5, 7
    st = stim.stimulus(ir, 5, np.arange(N), 0, T)
    d = oracle_lib.Design(ir)
    full = d.simulate(st, digest=True)
    for c in range(T):
        regs_next = d.simulate(st[:, :c + 1])["regs"]
        for s in range(N):
            acc = 0
            for j, v in enumerate(full["out"][s, c]):
                acc ^= oracle_lib.mix64(((j + 1) << 32) | int(v))
            for k, v in enumerate(regs_next[s]):
                acc ^= oracle_lib.mix64(((k + 1 + (1 << 31)) << 32) | int(v))
            assert acc == int(full["digest"][s, c])


def test_rejects_non_topological(oracle_lib):
    from rtlgen.builder import Builder
    b = Builder()
    x = b.input(4)
    y = b.op("NOT", 4, x)
    z = b.op("NOT", 4, y)
    ir = b.build()
    ir.ops = ir.ops[::-1].copy()
    with pytest.raises(ValueError):
        oracle_lib.Design(ir)
    del z
