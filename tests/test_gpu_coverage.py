"""Toggle coverage (N5, RTLSIM_F_COVERAGE) and the per-stimulus register
digest (rtlsim_reg_digest) against values computed from the CPU oracle's
register states: the oracle is stepped one cycle at a time (regs_in chaining)
so every R_c is known, coverage[k] = OR_{s,c} R_c[s][k] ^ R_{c+1}[s][k]; the
digest is DESIGN.md §3's register half, XOR_k mix(((k+1+2^31)<<32) | R[s][k])
(north star subsystem 4: the gathered per-stimulus results and coverage)."""
import numpy as np
import pytest

from rtlgen import designs, shaped, stim
from rtlgen.stim import _mix_np

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def R():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_icpp_linrzkh22_b200 import build, rtlsim
    build.build()
    return rtlsim


def oracle_states(oracle_lib, ir, st):
    """[T+1][N][RW] register states R_0 .. R_T, one oracle cycle at a time."""
    d = oracle_lib.Design(ir)
    N, T = st.shape[0], st.shape[1]
    r = np.tile(np.asarray(ir.reg_init, np.uint32), (N, 1))
    states = [r]
    for c in range(T):
        r = d.simulate(st[:, c:c + 1], regs_in=r, out=False, regs=True)["regs"]
        states.append(r)
    return np.stack(states)


def reg_digest_ref(regs):
    k = np.arange(regs.shape[1], dtype=np.uint64)
    z = ((k + np.uint64(1 + 0x80000000)) << np.uint64(32)) | regs.astype(np.uint64)
    with np.errstate(over="ignore"):
        return np.bitwise_xor.reduce(_mix_np(z), axis=1)


CASES = [
    ("tiny", 0, 70),                        # ragged N (padding stimuli masked)
    ("shaped2", 0, 45),
    ("shaped3-jit", 1, 64),
]


@pytest.mark.parametrize("kind,jit,N", CASES)
def test_coverage_and_reg_digest(R, oracle_lib, kind, jit, N):
    if kind == "tiny":
        ir = designs.tiny_dut()
        st = stim.tiny_stimulus(11, np.arange(N), 24, mode="B")
    else:
        ir = shaped.generate(2 if kind == "shaped2" else 3, scale=0.04)
        st = stim.stimulus(ir, 0x5150, np.arange(N), 0, 24)
    states = oracle_states(oracle_lib, ir, st)
    T = st.shape[1]
    flags = R.F_COVERAGE | (R.F_JIT if jit else 0)
    sim = R.Simulator(ir, chunk_cycles=10, flags=flags)
    sim.bind(st)
    assert not sim.coverage().any()                      # nothing simulated yet
    sim.run(T // 2, out=False, regs=False)
    want_half = np.bitwise_or.reduce(states[:T // 2] ^ states[1:T // 2 + 1], axis=(0, 1))
    assert np.array_equal(sim.coverage(), want_half)
    sim.run(T - T // 2, out=False, regs=False)
    want = np.bitwise_or.reduce(states[:-1] ^ states[1:], axis=(0, 1))
    assert np.array_equal(sim.coverage(clear=True), want)
    assert not sim.coverage().any()                      # cleared
    # register digest of the final state
    assert np.array_equal(sim.reg_digest(), reg_digest_ref(states[-1]))
    assert np.array_equal(sim.get_regs(), states[-1])
    if kind == "tiny":
        # the free-running parts toggle: the LFSR's 16 bits, the counter's low bits
        assert want.any()


def test_coverage_requires_flag(R):
    ir = designs.tiny_dut()
    sim = R.Simulator(ir)
    sim.bind(stim.tiny_stimulus(1, np.arange(8), 4))
    with pytest.raises(R.RtlsimError) as ei:
        sim.coverage()
    assert ei.value.code == -7
