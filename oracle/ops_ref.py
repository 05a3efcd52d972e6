"""Per-op mathematical definitions on Python arbitrary-precision ints.

TEST INFRASTRUCTURE ONLY. Each opcode is the definition of DESIGN.md §3
written with Python's own integer arithmetic (no word lanes, no carries, no
masks beyond the final ``mod 2^wd``), so it pins the C oracle's word-loop code
(oracle.c). Readings: two-state, IEEE 1364 context widths as
inherited through Verilator; truncation on assignment
(P:L648-651); shifts >= width give 0 / sign fill; DIVU/MODU by 0 give 0.
"""
from __future__ import annotations


def mask(w: int) -> int:
    return (1 << w) - 1


def signed(v: int, w: int) -> int:
    """Two's complement value of the w-bit pattern v."""
    v &= mask(w)
    return v - (1 << w) if v >> (w - 1) else v


def evaluate(name: str, wd: int, a: int = 0, wa: int = 0, b: int = 0, wb: int = 0,
             c: int = 0, wc: int = 0, imm: int = 0) -> int:
    a &= mask(wa) if wa else 0
    b &= mask(wb) if wb else 0
    c &= mask(wc) if wc else 0
    if name == "COPY":
        r = a
    elif name == "SEXT":
        r = signed(a, wa)
    elif name == "NOT":
        r = ~a                       # infinite-precision complement: bits above wa are 1
    elif name == "AND":
        r = a & b
    elif name == "OR":
        r = a | b
    elif name == "XOR":
        r = a ^ b
    elif name == "ADD":
        r = a + b
    elif name == "SUB":
        r = a - b
    elif name == "NEG":
        r = -a
    elif name == "MUL":
        assert max(wd, wa, wb) <= 64
        r = a * b
    elif name == "DIVU":
        assert max(wd, wa, wb) <= 64
        r = 0 if b == 0 else a // b
    elif name == "MODU":
        assert max(wd, wa, wb) <= 64
        r = 0 if b == 0 else a % b
    elif name in ("EQ", "NE", "LTU", "LEU", "GTU", "GEU"):
        r = {"EQ": a == b, "NE": a != b, "LTU": a < b, "LEU": a <= b,
             "GTU": a > b, "GEU": a >= b}[name]
    elif name in ("LTS", "LES", "GTS", "GES"):
        x, y = signed(a, wa), signed(b, wb)
        r = {"LTS": x < y, "LES": x <= y, "GTS": x > y, "GES": x >= y}[name]
    elif name == "SHL":
        r = 0 if b >= wd else a << b
    elif name == "SHRL":
        r = a >> b                   # b >= wa gives 0 automatically
    elif name == "SHRA":
        r = signed(a, wa) >> min(b, 4096)   # floor shift: sign fill when b >= width
    elif name == "MUX":
        r = b if a != 0 else c
    elif name == "CONCAT":
        r = (a << wb) | b
    elif name == "SLICE":
        assert imm + wd <= wa
        r = a >> imm
    elif name == "REDAND":
        r = a == mask(wa)
    elif name == "REDOR":
        r = a != 0
    elif name == "REDXOR":
        r = bin(a).count("1") & 1
    else:
        raise ValueError(name)
    return int(r) & mask(wd)
