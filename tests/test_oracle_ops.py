"""Pins for the oracle's per-op arithmetic (oracle.c EVAL) — CPU only.

Two kinds of pins:
* textbook/closed-form values that do not go through any of our code paths
  (carry chains, two's complement facts, Listing 2 of the paper, splitmix64's
  published first output), and
* the word-lane C code against Python's arbitrary-precision integers
  (oracle/ops_ref.py): exhaustive for widths <= 4, edge values and seeded
  random values for widths straddling every word boundary up to 1024.
"""
import itertools
import random

import pytest

from rtlgen import ir as I
from oracle import ops_ref

ALL = list(I.VALUE_OPS)   # MEMRD reads a memory: tests/test_oracle_mem.py


def ev(oracle_lib, name, wd, a=0, wa=0, b=0, wb=0, c=0, wc=0, imm=0):
    return oracle_lib.eval_op(I.OPCODES[name], wd, a, wa, b, wb, c, wc, imm)


# ---------------------------------------------------------- textbook pins --
def test_listing2_truncation(oracle_lib):
    """PAPER.md Listing 2: in[5:0] = 10'h1 + sum[13:0], truncated."""
    for s, want in [(0x3FFF, 0), (0x0005, 6), (0x003E, 0x3F), (0x003F, 0), (0x1234, (0x1234 + 1) & 0x3F)]:
        assert ev(oracle_lib, "ADD", 6, 1, 10, s, 14) == want


def test_wide_carry_chains(oracle_lib):
    for k in (1, 2, 3, 5, 32):
        w = 32 * k
        assert ev(oracle_lib, "ADD", w, (1 << w) - 1, w, 1, 1) == 0          # all-ones + 1 wraps
        assert ev(oracle_lib, "ADD", w + 1, (1 << w) - 1, w, 1, 1) == 1 << w  # carry out kept
        assert ev(oracle_lib, "SUB", w, 0, w, 1, 1) == (1 << w) - 1          # 0 - 1 borrows through
        assert ev(oracle_lib, "NEG", w, 1, w) == (1 << w) - 1
    assert ev(oracle_lib, "MUL", 64, (1 << 64) - 1, 64, 1, 1) == (1 << 64) - 1
    assert ev(oracle_lib, "MUL", 64, 1 << 32, 64, 1 << 32, 64) == 0             # 2^64 mod 2^64
    assert ev(oracle_lib, "MUL", 40, 0xFFFFF, 20, 0xFFFFF, 20) == (0xFFFFF * 0xFFFFF) & ((1 << 40) - 1)


def test_twos_complement_facts(oracle_lib):
    # -1 < 0 signed, but 0xFF > 0 unsigned
    assert ev(oracle_lib, "LTS", 1, 0xFF, 8, 0, 8) == 1
    assert ev(oracle_lib, "LTU", 1, 0xFF, 8, 0, 8) == 0
    # mixed widths: a 4-bit -1 equals an 8-bit -1 under sign extension, not under zero extension
    assert ev(oracle_lib, "GES", 1, 0xF, 4, 0xFF, 8) == 1 and ev(oracle_lib, "GTS", 1, 0xF, 4, 0xFF, 8) == 0
    assert ev(oracle_lib, "EQ", 1, 0xF, 4, 0xFF, 8) == 0
    # arithmetic shift right = floor division by 2^b of the signed value
    assert ev(oracle_lib, "SHRA", 8, 0x80, 8, 3, 4) == 0xF0      # -128 >> 3 = -16
    assert ev(oracle_lib, "SHRA", 8, 0x81, 8, 1, 4) == 0xC0      # -127 >> 1 = -64 (floor)
    assert ev(oracle_lib, "SHRA", 8, 0x80, 8, 200, 8) == 0xFF    # sign fill past the width
    assert ev(oracle_lib, "SHRA", 16, 0x80, 8, 4, 4) == 0xFFF8   # sign-extend to context width first
    assert ev(oracle_lib, "SEXT", 16, 0x80, 8) == 0xFF80
    assert ev(oracle_lib, "SEXT", 16, 0x7F, 8) == 0x007F


def test_context_width_rules(oracle_lib):
    # NOT of a 4-bit value into 8 bits: the zero-extended high bits invert to 1
    assert ev(oracle_lib, "NOT", 8, 0x5, 4) == 0xFA
    # shifts: amount >= width gives 0 (no C/PTX shift UB)
    assert ev(oracle_lib, "SHL", 32, 1, 32, 32, 6) == 0
    assert ev(oracle_lib, "SHL", 33, 1, 32, 32, 6) == 1 << 32      # context width = 33
    assert ev(oracle_lib, "SHRL", 32, 0xFFFFFFFF, 32, 32, 6) == 0
    assert ev(oracle_lib, "SHL", 8, 1, 8, 1 << 40, 41) == 0          # huge self-determined amount
    # division by zero gives 0 (Verilator's rule, reading 8)
    assert ev(oracle_lib, "DIVU", 16, 1234, 16, 0, 16) == 0
    assert ev(oracle_lib, "MODU", 16, 1234, 16, 0, 16) == 0
    assert ev(oracle_lib, "DIVU", 16, 1234, 16, 10, 16) == 123
    assert ev(oracle_lib, "MODU", 16, 1234, 16, 10, 16) == 4
    # concat / slice
    assert ev(oracle_lib, "CONCAT", 12, 0xA, 4, 0xBC, 8) == 0xABC
    assert ev(oracle_lib, "CONCAT", 8, 0xA, 4, 0xBC, 8) == 0xBC      # truncated
    assert ev(oracle_lib, "SLICE", 8, 0xABCDEF, 24, imm=8) == 0xCD
    assert ev(oracle_lib, "SLICE", 8, 0xAB << 60, 100, imm=60) == 0xAB  # across a word boundary
    # reductions
    assert ev(oracle_lib, "REDAND", 1, (1 << 100) - 1, 100) == 1
    assert ev(oracle_lib, "REDAND", 1, (1 << 100) - 2, 100) == 0
    assert ev(oracle_lib, "REDXOR", 1, 0b1011, 4) == 1
    assert ev(oracle_lib, "REDOR", 1, 1 << 99, 100) == 1
    # mux: any-width select, tested for non-zero
    assert ev(oracle_lib, "MUX", 8, 1 << 70, 71, 0x12, 8, 0x34, 8) == 0x12
    assert ev(oracle_lib, "MUX", 8, 0, 71, 0x12, 8, 0x34, 8) == 0x34


def test_mix64_published_vector(oracle_lib):
    """splitmix64 seeded with 0: first output 0xE220A8397B1DCDAF, second
    0x6E789E6AA1B965F4 (published reference sequence)."""
    g = 0x9E3779B97F4A7C15
    assert oracle_lib.mix64(g) == 0xE220A8397B1DCDAF
    assert oracle_lib.mix64(2 * g) == 0x6E789E6AA1B965F4


# ------------------------------------------ word lanes vs Python big ints --
def _operands(name):
    if name in I.UNARY and name != "SLICE":
        return 1
    if name == "MUX":
        return 3
    if name == "SLICE":
        return 1
    return 2


@pytest.mark.parametrize("name", ALL)
def test_exhaustive_small_widths(oracle_lib, name):
    """All operand values for widths 1..4 (shift amounts 0..7)."""
    n = _operands(name)
    widths = [1, 2, 3, 4]
    for wd, wa in itertools.product(widths, widths):
        if name == "SLICE":
            for lo in range(0, wa - wd + 1):
                for a in range(1 << wa):
                    assert ev(oracle_lib, name, wd, a, wa, imm=lo) == ops_ref.evaluate(name, wd, a, wa, imm=lo)
            continue
        if n == 1:
            for a in range(1 << wa):
                assert ev(oracle_lib, name, wd, a, wa) == ops_ref.evaluate(name, wd, a, wa)
            continue
        for wb in ([3] if name in I.SHIFTS else widths):
            if n == 2:
                for a in range(1 << wa):
                    for b in range(1 << wb):
                        got = ev(oracle_lib, name, wd, a, wa, b, wb)
                        assert got == ops_ref.evaluate(name, wd, a, wa, b, wb), (name, wd, wa, wb, a, b)
            else:
                for a in range(1 << wa):
                    for b in range(1 << wb):
                        for c in (0, 1, (1 << wb) - 1):
                            got = ev(oracle_lib, name, wd, a, wa, b, wb, c, wb)
                            assert got == ops_ref.evaluate(name, wd, a, wa, b, wb, c, wb)


BOUNDARY = [1, 5, 8, 15, 16, 17, 31, 32, 33, 63, 64, 65, 96, 127, 128, 129, 256, 512, 1000, 1024]


def _edges(w, rnd):
    m = (1 << w) - 1
    vals = {0, 1, m, 1 << (w - 1), (1 << (w - 1)) - 1 if w > 1 else 0}
    vals.add(rnd.getrandbits(w))
    vals.add(rnd.getrandbits(w))
    return sorted(v & m for v in vals)


@pytest.mark.parametrize("name", ALL)
def test_word_boundaries(oracle_lib, name):
    rnd = random.Random(0xC0FFEE + I.OPCODES[name])
    n = _operands(name)
    ws = [w for w in BOUNDARY if (w <= 64 or name not in I.MULDIV)]
    for _ in range(160):
        wd, wa, wb = rnd.choice(ws), rnd.choice(ws), rnd.choice(ws)
        if name in I.SHIFTS:
            wb = rnd.choice([3, 6, 11, 32, 33, 40])
        if name == "SLICE":
            wd = rnd.randint(1, wa)
            lo = rnd.randint(0, wa - wd)
            for a in _edges(wa, rnd):
                assert ev(oracle_lib, name, wd, a, wa, imm=lo) == ops_ref.evaluate(name, wd, a, wa, imm=lo)
            continue
        for a in _edges(wa, rnd):
            if n == 1:
                assert ev(oracle_lib, name, wd, a, wa) == ops_ref.evaluate(name, wd, a, wa)
                continue
            bvals = _edges(wb, rnd)
            if name in I.SHIFTS:
                bvals = sorted(x for x in {0, 1, wd - 1, wd, wd + 1, wa - 1, wa, wa + 1,
                                           (1 << wb) - 1, rnd.getrandbits(wb)} if x < (1 << wb))
            for b in bvals:
                b &= (1 << wb) - 1
                if n == 2:
                    got = ev(oracle_lib, name, wd, a, wa, b, wb)
                    assert got == ops_ref.evaluate(name, wd, a, wa, b, wb), (name, wd, wa, wb, a, b)
                else:
                    c = rnd.getrandbits(wb)
                    got = ev(oracle_lib, name, wd, a, wa, b, wb, c, wb)
                    assert got == ops_ref.evaluate(name, wd, a, wa, b, wb, c, wb)
