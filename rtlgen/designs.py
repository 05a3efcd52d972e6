"""Hand-built designs: the tiny DUT of config 1, small pin fixtures and random
combinational / sequential DAGs for brute-force and invariant tests.

Input plumbing only (no evaluation). SURVEY §8(d) config 1: "8-bit counter
(en, rst), 4-bit ALU (op[2:0], a[3:0], b[3:0] -> y[3:0], carry, zero), 16-bit
Fibonacci LFSR (init 0xACE1), RED_XOR parity".
"""
from __future__ import annotations

import numpy as np

from . import ir as I
from .builder import Builder

LFSR_INIT = 0xACE1

# tiny DUT stimulus word order (IW = 5): rst, en, op, a, b
TINY_INPUTS = ("rst", "en", "op", "a", "b")
# output word order (OW = 8)
TINY_OUTPUTS = ("cnt", "y", "carry", "zero", "y_q", "lfsr", "parity", "acc")


def tiny_dut() -> I.IR:
    """Config 1: counter + ALU + LFSR + parity (+ a 40-bit accumulator so the
    tiny design also crosses the 32-bit word boundary)."""
    b = Builder("tiny")
    rst = b.input(1, "rst")
    en = b.input(1, "en")
    op = b.input(3, "op")
    a = b.input(4, "a")
    bb = b.input(4, "b")

    # 8-bit counter: cnt' = rst ? 0 : (en ? cnt + 1 : cnt)
    cnt = b.reg(8, 0, "cnt")
    one8 = b.const(8, 1)
    zero8 = b.const(8, 0)
    inc = b.ADD(8, cnt, one8)
    t = b.MUX(8, en, inc, cnt)
    b.set_d(cnt, b.MUX(8, rst, zero8, t))

    # 4-bit ALU, op: 0 ADD 1 SUB 2 AND 3 OR 4 XOR 5 SHL b[1:0] 6 SHR b[1:0] 7 NOT a
    sum5 = b.ADD(5, a, bb)
    carry = b.slice(sum5, 4, 1)
    r_add = b.COPY(4, sum5)
    r_sub = b.SUB(4, a, bb)
    r_and = b.AND(4, a, bb)
    r_or = b.OR(4, a, bb)
    r_xor = b.XOR(4, a, bb)
    sh = b.slice(bb, 0, 2)
    r_shl = b.SHL(4, a, sh)
    r_shr = b.SHRL(4, a, sh)
    r_not = b.NOT(4, a)
    op0 = b.slice(op, 0, 1)
    op1 = b.slice(op, 1, 1)
    op2 = b.slice(op, 2, 1)
    m01 = b.MUX(4, op0, r_sub, r_add)
    m23 = b.MUX(4, op0, r_or, r_and)
    m45 = b.MUX(4, op0, r_shl, r_xor)
    m67 = b.MUX(4, op0, r_not, r_shr)
    m03 = b.MUX(4, op1, m23, m01)
    m47 = b.MUX(4, op1, m67, m45)
    y = b.MUX(4, op2, m47, m03)
    zero4 = b.const(4, 0)
    zero = b.EQ(1, y, zero4)
    y_q = b.reg(4, 0, "y_q")
    b.set_d(y_q, y)

    # 16-bit Fibonacci LFSR x^16+x^14+x^13+x^11+1, right shift, taps 0,2,3,5
    lfsr = b.reg(16, LFSR_INIT, "lfsr")
    t0 = b.slice(lfsr, 0, 1)
    t2 = b.slice(lfsr, 2, 1)
    t3 = b.slice(lfsr, 3, 1)
    t5 = b.slice(lfsr, 5, 1)
    fb = b.XOR(1, b.XOR(1, t0, t2), b.XOR(1, t3, t5))
    nxt = b.CONCAT(16, fb, b.slice(lfsr, 1, 15))
    init = b.const(16, LFSR_INIT)
    b.set_d(lfsr, b.MUX(16, rst, init, nxt))
    parity = b.REDXOR(1, lfsr)

    # 40-bit accumulator: acc' = rst ? 0 : acc + ({cnt, y, a} << 20)
    acc = b.reg(40, 0, "acc")
    cat = b.CONCAT(16, b.CONCAT(12, cnt, y), a)
    sh20 = b.const(5, 20)
    acc_sum = b.ADD(40, acc, b.SHL(40, cat, sh20))
    zero40 = b.const(40, 0)
    b.set_d(acc, b.MUX(40, rst, zero40, acc_sum))

    for s in (cnt, y, carry, zero, y_q, lfsr, parity, acc):
        b.output(s)
    return b.build()


def swap_dut() -> I.IR:
    """Non-blocking register update (reading 16c): a<=b; b<=a swaps;
    a 3-stage shift chain s0<=in, s1<=s0, s2<=s1 delays by exactly 3."""
    b = Builder("swap")
    x = b.input(7, "x")
    ra = b.reg(7, 0x15, "ra")
    rb = b.reg(7, 0x6A, "rb")
    b.set_d(ra, rb)
    b.set_d(rb, ra)
    s0 = b.reg(7, 0, "s0")
    s1 = b.reg(7, 0, "s1")
    s2 = b.reg(7, 0, "s2")
    b.set_d(s0, x)
    b.set_d(s1, s0)
    b.set_d(s2, s1)
    for s in (ra, rb, s2):
        b.output(s)
    return b.build()


def listing2_dut() -> I.IR:
    """PAPER.md Listing 2: ``c1.in = 10'h1 + c1.sum`` with a
    6-bit ``in`` and a 14-bit ``sum`` — truncation on assignment."""
    b = Builder("listing2")
    s = b.input(14, "sum")
    one = b.const(10, 1)
    res = b.ADD(6, one, s, out_name="in")
    b.output(res)
    return b.build()


# ------------------------------------------------------------- random DAGs --
_WIDTHS = [1, 2, 3, 4, 5, 7, 8, 9, 15, 16, 17, 31, 32, 33, 47, 63, 64, 65, 96, 100, 127, 128, 129, 200, 256]


def random_dag(seed: int, n_ops: int = 100, input_widths=(3, 5, 1, 4, 3),
               n_regs: int = 0, n_partitions: int = 1, n_consts: int = 6,
               max_width: int = 256, outputs: str = "all") -> I.IR:
    """Random DAG over all opcodes. Operands pick any earlier signal (any
    width); widths straddle every 32-bit word boundary up to ``max_width``.
    Partitions are contiguous op ranges assigned in a shuffled order so the
    partition DAG is acyclic but not numerically ordered."""
    rng = np.random.default_rng(seed)
    b = Builder(f"dag{seed}")
    widths = [w for w in _WIDTHS if w <= max_width]
    pool: list[int] = []
    for w in input_widths:
        pool.append(b.input(int(w)))
    for _ in range(n_consts):
        w = int(rng.choice(widths))
        v = int.from_bytes(rng.bytes((w + 7) // 8), "little") & ((1 << w) - 1)
        if rng.random() < 0.3:
            v = int(rng.integers(0, 8))          # small shift amounts / selects
        pool.append(b.const(w, v))
    regs = []
    for _ in range(n_regs):
        w = int(rng.choice(widths))
        init = int.from_bytes(rng.bytes((w + 7) // 8), "little") & ((1 << w) - 1)
        q = b.reg(w, init)
        regs.append(q)
        pool.append(q)
    names = list(I.VALUE_OPS)
    order = list(range(n_partitions))
    rng.shuffle(order)
    comb = []
    for i in range(n_ops):
        b.partition(order[min(n_partitions - 1, i * n_partitions // max(1, n_ops))])
        name = str(rng.choice(names))
        wd = int(rng.choice(widths))

        def pick(maxw=None):
            cand = pool if maxw is None else [s for s in pool if b.width[s] <= maxw]
            if not cand:
                cand = pool
            # bias towards recent values so DAGs get deep
            if rng.random() < 0.6 and len(cand) > 4:
                return int(cand[-1 - int(rng.integers(0, min(len(cand), 8)))])
            return int(cand[int(rng.integers(0, len(cand)))])

        if name in I.MULDIV:
            wd = min(wd, 64)
            a, bo = pick(64), pick(64)
            if b.width[a] > 64 or b.width[bo] > 64:
                name = "AND"
            d = b.op(name, wd, a, bo)
        elif name in I.COMPARES:
            d = b.op(name, int(rng.choice([1, 1, 1, 3])), pick(), pick())
        elif name in I.REDUCTIONS:
            d = b.op(name, int(rng.choice([1, 1, 2])), pick())
        elif name == "SLICE":
            a = pick()
            wa = b.width[a]
            wd = int(rng.integers(1, wa + 1))
            lo = int(rng.integers(0, wa - wd + 1))
            d = b.op("SLICE", wd, a, imm=lo)
        elif name == "MUX":
            d = b.op("MUX", wd, pick(), pick(), pick())
        elif name in ("NOT", "NEG", "COPY", "SEXT"):
            d = b.op(name, wd, pick())
        elif name == "CONCAT":
            a, bo = pick(), pick()
            wd = min(max_width, b.width[a] + b.width[bo]) if rng.random() < 0.7 else wd
            d = b.op(name, wd, a, bo)
        elif name in I.SHIFTS:
            sh = pick(16) if rng.random() < 0.8 else pick()
            d = b.op(name, wd, pick(), sh)
        else:
            d = b.op(name, wd, pick(), pick())
        comb.append(d)
        pool.append(d)
    for q in regs:
        b.set_d(q, int(comb[-1 - int(rng.integers(0, min(len(comb), 20)))]) if comb else q)
    if outputs == "all":
        for s in comb:
            b.output(s)
        for q in regs:
            b.output(q)
    else:
        for s in comb[-int(outputs):]:
            b.output(s)
    return b.build()


def exhaustive_stimulus(ir: I.IR) -> np.ndarray:
    """[2^bits][1][IW]: stimulus s enumerates every input combination (bit
    fields of s in input order). Requires total input bits <= 20."""
    widths = [int(ir.width[s]) for s in ir.input_sig]
    total = sum(widths)
    assert total <= 20
    n = 1 << total
    s = np.arange(n, dtype=np.uint64)
    cols = []
    sh = 0
    for w in widths:
        v = (s >> np.uint64(sh)) & np.uint64((1 << w) - 1)
        cols.append(v.astype(np.uint32))
        for _ in range(I.nwords(w) - 1):
            cols.append(np.zeros(n, dtype=np.uint32))
        sh += w
    return np.stack(cols, axis=1).reshape(n, 1, -1)


# ------------------------------------------------------------- memories --
# ARRSEL (§3.1.1, Fig 5): an array variable read at a run-time index,
# written by synchronous ports (reading 12).
MEMSEQ_INIT = [100 + i for i in range(8)]


def mem_seq_dut() -> I.IR:
    """Free-running 8-bit counter c; 8 x 8-bit memory; each cycle writes
    c + 1 at entry c mod 8 and reads entry (c - 1) mod 8 (rd_prev) and entry
    c mod 8 (rd_same, read-during-write). Closed forms (oracle pins):
    rd_prev_c = c for c >= 1 (107 at c = 0); rd_same_c = c - 7 for c >= 8
    (100 + c before): a read sees the memory as it was before the edge."""
    b = Builder("memseq")
    c = b.reg(8, 0, "c")
    one = b.const(8, 1)
    c1 = b.ADD(8, c, one)
    b.set_d(c, c1)
    m = b.mem(8, 8, MEMSEQ_INIT)
    wa = b.slice(c, 0, 3)
    cm1 = b.SUB(8, c, one)
    ra = b.slice(cm1, 0, 3)
    en = b.const(1, 1)
    b.wport(m, wa, c1, en)
    b.output(c)
    b.output(b.memrd(m, ra, "rd_prev"))
    b.output(b.memrd(m, wa, "rd_same"))
    return b.build()


MEMB_DEPTH = 5
MEMB_INIT = [0x1111 * (i + 1) for i in range(MEMB_DEPTH)]


def mem_bounds_dut() -> I.IR:
    """Inputs we, waddr[2:0], wdata[15:0], raddr[2:0]; a 5 x 16-bit memory.
    Entries 5..7 do not exist: writes there are ignored, reads return 0."""
    b = Builder("membounds")
    we = b.input(1, "we")
    waddr = b.input(3, "waddr")
    wdata = b.input(16, "wdata")
    raddr = b.input(3, "raddr")
    m = b.mem(16, MEMB_DEPTH, MEMB_INIT)
    b.wport(m, waddr, wdata, we)
    b.output(b.memrd(m, raddr, "rdata"))
    return b.build()


def mem_two_port_dut() -> I.IR:
    """Two write ports hit the same entry every cycle (the counter's low 2
    bits): port 0 writes c, port 1 writes ~c — the later port wins, so
    rd_prev (entry (c - 1) mod 4) = ~(c - 1) for c >= 1."""
    b = Builder("mem2p")
    c = b.reg(8, 0, "c")
    one = b.const(8, 1)
    b.set_d(c, b.ADD(8, c, one))
    m = b.mem(8, 4)
    wa = b.slice(c, 0, 2)
    en = b.const(1, 1)
    b.wport(m, wa, c, en)
    b.wport(m, wa, b.NOT(8, c), en)
    ra = b.slice(b.SUB(8, c, one), 0, 2)
    b.output(c)
    b.output(b.memrd(m, ra, "rd_prev"))
    return b.build()


def regfile_dut(seed: int = 7, depth: int = 32, width: int = 32, n_read: int = 2, wide: int = 72,
                parts: int = 1) -> I.IR:
    """A register-file-heavy design: a depth x width memory with n_read read
    ports and one write port driven from inputs, a depth/4 x `wide`-bit
    memory (three-word entries) and a 16 x 1-bit memory, each read value
    mixed through a little logic into registers and outputs; addresses are one
    bit wider than needed (out-of-range reads and writes occur)."""
    rng = np.random.default_rng(seed)
    b = Builder("regfile")
    aw = int(np.ceil(np.log2(depth))) + 1
    we = b.input(1, "we")
    waddr = b.input(aw, "waddr")
    wdata = b.input(width, "wdata")
    raddrs = [b.input(aw, f"raddr{i}") for i in range(n_read)]
    m = b.mem(width, depth, [int(x) for x in rng.integers(0, 1 << min(width, 62), size=depth)])
    b.wport(m, waddr, wdata, we)
    acc = b.reg(width, 0, "acc")
    vals = []
    for i, ra in enumerate(raddrs):
        if parts > 1:
            b.partition(i % parts)
        v = b.memrd(m, ra)
        vals.append(v)
        b.output(v)
    s = b.ADD(width, vals[0], vals[-1])
    b.set_d(acc, b.XOR(width, acc, s))
    b.output(acc)
    # a wide memory (entries of 3 words) written with {wdata, wdata, waddr}
    dw = max(4, depth // 4)
    mw = b.mem(wide, dw, [int(x) for x in rng.integers(0, 1 << 62, size=dw)])
    aw2 = int(np.ceil(np.log2(dw))) + 1
    wa2 = b.slice(waddr, 0, min(aw, aw2))
    cat = b.CONCAT(wide, b.CONCAT(2 * width, wdata, wdata), waddr)
    b.wport(mw, wa2, cat, we)
    b.output(b.memrd(mw, b.slice(raddrs[0], 0, min(aw, aw2))))
    # a 1-bit memory
    m1 = b.mem(1, 16, [int(x) for x in rng.integers(0, 2, size=16)])
    b.wport(m1, b.slice(waddr, 0, 4), b.slice(wdata, 0, 1), we)
    r1 = b.memrd(m1, b.slice(raddrs[-1], 0, 4))
    f = b.reg(1, 0, "f")
    b.set_d(f, b.XOR(1, f, r1))
    b.output(r1)
    b.output(f)
    return b.build()
