"""TMEM schedules (r2): U32 values computed by ops live in
tensor memory (tcgen05.ld / tcgen05.st, one TMEM lane per stimulus), four
tiles per CTA on the four lane quarters. Forced on (RTLSIM_JIT_TMEM=1) for
designs the auto choice would leave classic, and compared bit for bit with
the CPU oracle: every output, register and per-cycle digest; wide values up
to 1024 bits (vector tcgen05 runs), several partitions, ragged N (N_pad in
128s), memories, run splitting, the check-mode digest kernels, M1 cycle
loop. Config 4's full-size tests (test_gpu_fullsize / test_gpu_golden) run
the TMEM schedule through the auto choice."""
import numpy as np
import pytest

from rtlgen import designs, shaped, stim

pytestmark = pytest.mark.gpu


@pytest.fixture(scope="module")
def R():
    import torch
    assert torch.cuda.is_available(), "GPU tests need a CUDA device"
    from paper_conf_icpp_linrzkh22_b200 import build, rtlsim
    build.build()
    return rtlsim


@pytest.fixture(autouse=True)
def tmem_on(monkeypatch):
    monkeypatch.setenv("RTLSIM_JIT_TMEM", "1")


def _same(got, want, what):
    for k in ("out", "regs", "digest"):
        if want.get(k) is None or got.get(k) is None:
            continue
        a, b = got[k], want[k]
        assert a.shape == b.shape, (what, k)
        if not np.array_equal(a, b):
            bad = np.argwhere(a != b)
            raise AssertionError(f"{what}: {k} differs at {len(bad)} places, first {bad[:5].tolist()}")


def _run(R, ir, st, cycles=None, **opt):
    sim = R.Simulator(ir, flags=R.F_JIT | opt.pop("flags", 0), **opt)
    assert sim.stats()["tmem_cols"] > 0, "TMEM schedule not chosen"
    sim.bind(st)
    return sim, sim.run(cycles or st.shape[1], out=True, regs=True, digest=True)


@pytest.mark.parametrize("seed,parts", [(0, 1), (1, 3), (2, 5), (3, 2)])
def test_tmem_wide_partitioned(R, oracle_lib, seed, parts):
    ir = designs.random_dag(500 + seed, n_ops=300, n_regs=24, n_partitions=parts,
                            input_widths=(7, 33, 1, 64, 100), max_width=1024)
    st = stim.stimulus(ir, 11 + seed, np.arange(96), 0, 40, mask=False)
    _, got = _run(R, ir, st, chunk_cycles=7)
    _same(got, oracle_lib.simulate(ir, st, digest=True, threads=8), f"seq{seed}/{parts}")


@pytest.mark.parametrize("cid,scale,N,T", [(2, 1.0, 200, 40), (3, 0.25, 160, 24), (4, 0.02, 129, 8)])
def test_tmem_shaped(R, oracle_lib, cid, scale, N, T):
    ir = shaped.generate(cid, scale=scale)
    st = stim.stimulus(ir, stim.STIM_SEED_BASE + cid, np.arange(N), 0, T)
    _, got = _run(R, ir, st, chunk_cycles=16)
    _same(got, oracle_lib.simulate(ir, st, digest=True, threads=16), f"config{cid}@{scale}")


@pytest.mark.parametrize("lanes", [1, 3, 8])
def test_tmem_lanes_ragged(R, oracle_lib, lanes):
    ir = designs.random_dag(77, n_ops=400, n_regs=30, n_partitions=3, input_widths=(9, 40, 1, 70),
                            max_width=300)
    for N in (1, 33, 130):
        st = stim.stimulus(ir, 5 + N, np.arange(N), 0, 20, mask=False)
        _, got = _run(R, ir, st, chunk_cycles=6, op_lanes=lanes)
        _same(got, oracle_lib.simulate(ir, st, digest=True, threads=8), f"L={lanes} N={N}")


def test_tmem_run_splitting(R, oracle_lib):
    ir = shaped.generate(4, scale=0.02)
    st = stim.stimulus(ir, 0x7E, np.arange(64), 0, 20)
    want = oracle_lib.simulate(ir, st, digest=True, threads=16)
    sim = R.Simulator(ir, chunk_cycles=3, flags=R.F_JIT)
    sim.bind(st)
    a = sim.run(7, out=True, regs=False, digest=True)
    b = sim.run(13, out=True, regs=True, digest=True)
    assert np.array_equal(np.concatenate([a["out"], b["out"]], axis=1), want["out"])
    assert np.array_equal(np.concatenate([a["digest"], b["digest"]], axis=1), want["digest"])
    assert np.array_equal(b["regs"], want["regs"])


def test_tmem_regfile(R, oracle_lib):
    ir = designs.regfile_dut(seed=2, depth=32, width=64, n_read=3, parts=2)
    st = stim.stimulus(ir, 0x5EED, np.arange(130), 0, 50)
    want = oracle_lib.Design(ir).simulate(st, digest=True, mems=True, threads=8)
    sim, got = _run(R, ir, st, chunk_cycles=16)
    _same(got, want, "regfile")
    assert np.array_equal(sim.get_mems(), want["mems"])
