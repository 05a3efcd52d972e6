"""Pins for the oracle's cycle semantics on hand-built designs — CPU only.

Every expected value here comes from a closed form, a textbook sequence or
the paper's worked example, computed directly with numpy / Python integers —
never from the simulator under test (SURVEY §8(c) pin table).
"""
import numpy as np
import pytest

from rtlgen import designs, stim
from rtlgen import ir as I

T_TINY = 100


def _fields(out, ir):
    """Split out[N][T][OW] into named integer arrays (outputs are <= 64 bits)."""
    res = {}
    k = 0
    names = designs.TINY_OUTPUTS
    for name, s in zip(names, ir.output_sig):
        n = I.nwords(int(ir.width[s]))
        v = np.zeros(out.shape[:2], dtype=np.uint64)
        for t in range(n):
            v |= out[..., k + t].astype(np.uint64) << np.uint64(32 * t)
        res[name] = v
        k += n
    return res


def _prefix_window(rst, en):
    """count[c] = sum of en over [l(c), c), l(c) = 1 + last c' < c with rst=1 (else 0)."""
    N, T = rst.shape
    cnt = np.zeros((N, T), np.int64)
    run = np.zeros(N, np.int64)
    for c in range(T):
        cnt[:, c] = run
        run = np.where(rst[:, c] == 1, 0, run + en[:, c])
    return cnt


@pytest.fixture(scope="module")
def tiny():
    return designs.tiny_dut()


def test_tiny_shape(tiny):
    s = tiny.summary()
    assert 40 <= s["n_ops"] <= 80, s
    assert tiny.IW == 5 and tiny.n_regs == 4


def test_counter_free_run(oracle_lib, tiny):
    """Mode A (rst=0, en=1): O_c = c mod 256 (pre-edge sampling); final reg = T mod 256."""
    N = 64
    st = stim.tiny_stimulus(1, np.arange(N), 300, mode="A")
    r = oracle_lib.simulate(tiny, st)
    f = _fields(r["out"], tiny)
    c = np.arange(300)
    assert np.array_equal(f["cnt"], np.broadcast_to(c % 256, (N, 300)))
    assert np.all(r["regs"][:, 0] == 300 % 256)


def test_counter_en_rst_closed_form(oracle_lib, tiny):
    N = 256
    st = stim.tiny_stimulus(7, np.arange(N), T_TINY, mode="B")
    r = oracle_lib.simulate(tiny, st)
    f = _fields(r["out"], tiny)
    rst, en = st[..., 0].astype(np.int64), st[..., 1].astype(np.int64)
    assert rst.any() and (1 - rst).any() and en.any()
    want = _prefix_window(rst, en) % 256
    assert np.array_equal(f["cnt"].astype(np.int64), want)


def test_alu_all_combinations(oracle_lib, tiny):
    """All 16 x 16 x 8 = 2048 (a, b, op) combinations appear (enumeration index);
    y = textbook result mod 16, carry = bit 4 of a + b, zero = (y == 0), and the
    registered y_q at cycle c equals y at c - 1 (0 at c = 0)."""
    N, T = 64, 32      # 2048 (s, c) pairs = every combination exactly once
    st = stim.tiny_stimulus(3, np.arange(N), T, mode="B")
    r = oracle_lib.simulate(tiny, st)
    f = _fields(r["out"], tiny)
    op, a, b = (st[..., 2].astype(np.int64), st[..., 3].astype(np.int64), st[..., 4].astype(np.int64))
    assert len(set(zip(op.ravel(), a.ravel(), b.ravel()))) == 2048
    sh = b & 3
    table = [a + b, a - b, a & b, a | b, a ^ b, a << sh, a >> sh, ~a]
    y = np.choose(op, table) & 15
    assert np.array_equal(f["y"].astype(np.int64), y)
    assert np.array_equal(f["carry"].astype(np.int64), ((a + b) >> 4) & 1)
    assert np.array_equal(f["zero"].astype(np.int64), (y == 0).astype(np.int64))
    yq = np.concatenate([np.zeros((N, 1), np.int64), y[:, :-1]], axis=1)
    assert np.array_equal(f["y_q"].astype(np.int64), yq)


def _lfsr_step(x):
    # Fibonacci LFSR x^16 + x^14 + x^13 + x^11 + 1 (textbook form)
    bit = ((x >> 0) ^ (x >> 2) ^ (x >> 3) ^ (x >> 5)) & 1
    return (x >> 1) | (bit << 15)


def test_lfsr_textbook_sequence_and_period(oracle_lib, tiny):
    seq = [0xACE1]
    for _ in range(65536):
        seq.append(_lfsr_step(seq[-1]))
    # published first states of this textbook LFSR, and its maximal period
    assert seq[:10] == [0xACE1, 0x5670, 0xAB38, 0x559C, 0x2ACE, 0x1567, 0x8AB3, 0x4559, 0x22AC, 0x9156]
    assert seq[65535] == 0xACE1 and 0xACE1 not in seq[1:65535]
    N = 4
    st = stim.tiny_stimulus(1, np.arange(N), 200, mode="A")
    f = _fields(oracle_lib.simulate(tiny, st)["out"], tiny)
    assert np.array_equal(f["lfsr"][0], np.asarray(seq[:200], np.uint64))
    par = np.array([bin(x).count("1") & 1 for x in seq[:200]], np.uint64)
    assert np.array_equal(f["parity"][0], par)


def test_lfsr_full_period_through_simulator(oracle_lib, tiny):
    """After exactly T = 65535 rising edges the maximal-length LFSR is back at
    0xACE1 (and the free-running counter at 65535 mod 256)."""
    T = 65535
    st = stim.tiny_stimulus(1, [0], T, mode="A")
    r = oracle_lib.simulate(tiny, st, out=False)
    # register words: cnt(1) y_q(1) lfsr(1) acc(2)
    assert int(r["regs"][0, 2]) == 0xACE1
    assert int(r["regs"][0, 0]) == T % 256


def test_lfsr_with_reset(oracle_lib, tiny):
    N = 32
    st = stim.tiny_stimulus(11, np.arange(N), T_TINY, mode="B")
    f = _fields(oracle_lib.simulate(tiny, st)["out"], tiny)
    rst = st[..., 0].astype(np.int64)
    seq = [0xACE1]
    for _ in range(T_TINY):
        seq.append(_lfsr_step(seq[-1]))
    steps = _prefix_window(rst, np.ones_like(rst))
    want = np.asarray(seq, np.uint64)[steps]
    assert np.array_equal(f["lfsr"], want)


def test_accumulator_40bit(oracle_lib, tiny):
    """acc' = rst ? 0 : acc + ({cnt, y, a} << 20), mod 2^40."""
    N = 16
    T = 400
    st = stim.tiny_stimulus(5, np.arange(N), T, mode="A")
    f = _fields(oracle_lib.simulate(tiny, st)["out"], tiny)
    cat = (f["cnt"].astype(object) << 8) | (f["y"].astype(object) << 4) | st[..., 3].astype(object)
    acc = np.zeros((N, T), object)
    run = np.zeros(N, object)
    for c in range(T):
        acc[:, c] = run
        run = (run + (cat[:, c] << 20)) % (1 << 40)
    assert np.array_equal(f["acc"].astype(object), acc)
    assert (f["acc"] >= (1 << 32)).any()     # the 40-bit value really crosses a word


def test_swap_and_shift_chain(oracle_lib):
    """Non-blocking update: a<=b; b<=a swaps every cycle; s2 = x delayed by 3."""
    ir = designs.swap_dut()
    N, T = 8, 20
    st = stim.stimulus(ir, 9, np.arange(N), 0, T)
    out = oracle_lib.simulate(ir, st)["out"]
    ra, rb, s2 = out[..., 0], out[..., 1], out[..., 2]
    even = (np.arange(T) % 2) == 0
    assert np.all(ra[:, even] == 0x15) and np.all(ra[:, ~even] == 0x6A)
    assert np.all(rb[:, even] == 0x6A) and np.all(rb[:, ~even] == 0x15)
    x = st[..., 0]
    assert np.all(s2[:, :3] == 0) and np.array_equal(s2[:, 3:], x[:, :-3])


def test_listing2_design(oracle_lib):
    """PAPER.md Listing 2 as a one-op design: in = 10'h1 + sum, 6-bit result."""
    ir = designs.listing2_dut()
    vals = np.array([0x3FFF, 0x0005, 0x003F, 0x1234, 0], np.uint32)
    st = vals.reshape(-1, 1, 1)
    out = oracle_lib.simulate(ir, st)["out"][:, 0, 0]
    assert list(out) == [0, 6, 0, (0x1234 + 1) & 0x3F, 1]


def test_input_bits_above_width_ignored(oracle_lib, tiny):
    """Reading 15: stimulus bits above an input's width are masked."""
    N, T = 32, 50
    st = stim.tiny_stimulus(2, np.arange(N), T, mode="B")
    noisy = st | (np.uint32(0xFFFFFFF0) << np.uint32(0))
    noisy = np.where(np.arange(5) < 2, st | np.uint32(0xFFFFFFFE), noisy).astype(np.uint32)
    noisy[..., 2] = st[..., 2] | np.uint32(0xFFFFFFF8)
    a = oracle_lib.simulate(tiny, st, digest=True)
    b = oracle_lib.simulate(tiny, noisy, digest=True)
    assert np.array_equal(a["out"], b["out"]) and np.array_equal(a["digest"], b["digest"])
