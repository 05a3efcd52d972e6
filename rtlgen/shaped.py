"""Seeded "shaped" synthetic designs for configs 2-4.

The real benchmarks of the paper (riscv-mini, Spinal/VexRiscv, NVDLA hw_small;
P:L967-971) are not available offline, so these generators produce levelized
designs with the op mix, width mix, register fraction, partition structure
and fan-in locality SURVEY §8(d) fixes. The parameters below were FIXED
before any kernel tuning and must not be retuned to hit a target.

Input plumbing only: it draws a graph; it evaluates nothing.
"""
from __future__ import annotations

import dataclasses

import numpy as np

from . import ir as I
from .stim import DESIGN_SEED_BASE

# width classes: (lo, hi) inclusive
CLASSES = [(1, 1), (2, 8), (9, 16), (17, 32), (33, 64), (65, 128), (129, 512)]
NCLS = len(CLASSES)

# op mix: 30% logic, 20% MUX, 10% arith, 12% compares,
# 20% CONCAT/SLICE/ZEXT/SEXT, 4% shifts, 3% reductions, 1% MUL/DIVU/MODU
OP_MIX = {
    "AND": 9, "OR": 9, "XOR": 7, "NOT": 5,
    "MUX": 20,
    "ADD": 5, "SUB": 4, "NEG": 1,
    "EQ": 4, "NE": 2, "LTU": 2, "LEU": 1, "GTU": 1, "GEU": 0.5,
    "LTS": 0.375, "LES": 0.375, "GTS": 0.375, "GES": 0.375,
    "CONCAT": 6, "SLICE": 8, "COPY": 3, "SEXT": 3,
    "SHL": 2, "SHRL": 1.5, "SHRA": 0.5,
    "REDAND": 1, "REDOR": 1, "REDXOR": 1,
    "MUL": 0.6, "DIVU": 0.2, "MODU": 0.2,
}


@dataclasses.dataclass
class Shape:
    name: str
    config_id: int
    n_ops: int
    n_partitions: int
    levels_per_partition: int
    width_dist: list            # per class probability (len NCLS)
    exact32: float = 0.0        # fraction of class-3 widths forced to exactly 32
    reg_fraction: float = 0.1
    input_widths: tuple = ()
    n_outputs: int = 8
    partition_width: int = 1    # partitions per partition-DAG level
    p_reg: float = 0.15         # operand source probabilities
    p_in: float = 0.03
    p_const: float = 0.05
    p_xpart: float = 0.0
    back_probs: tuple = (0.5, 0.25, 0.15, 0.10)   # operand from level l-1..l-4
    same_class: float = 0.8
    const_fraction: float = 0.01
    regbank: bool = False


SHAPES = {
    2: Shape("riscv-mini-shaped", 2, 10_000, 1, 40,
             # 45% 32-bit, 35% 1-bit, 15% 2-8, 5% 9-16
             [0.35, 0.15, 0.05, 0.45, 0.0, 0.0, 0.0], exact32=1.0,
             reg_fraction=0.10, input_widths=(32, 32, 16, 8, 5, 5, 1, 1), n_outputs=8,
             regbank=True),
    3: Shape("spinal-shaped", 3, 50_000, 8, 40,
             [0.40, 0.15, 0.05, 0.38, 0.02, 0.0, 0.0],
             reg_fraction=0.10, n_outputs=16, partition_width=2, p_xpart=0.02),
    4: Shape("nvdla-shaped", 4, 1_048_576, 64, 64,
             [0.40, 0.20, 0.15, 0.12, 0.06, 0.04, 0.03],
             reg_fraction=0.125, n_outputs=64, partition_width=8, p_xpart=0.02),
}
_N_INPUTS = {2: 8, 3: 16, 4: 64}


def _sample_widths(rng, n, dist, exact32=0.0):
    cls = rng.choice(NCLS, size=n, p=np.asarray(dist) / np.sum(dist))
    lo = np.array([c[0] for c in CLASSES])[cls]
    hi = np.array([c[1] for c in CLASSES])[cls]
    w = lo + (rng.random(n) * (hi - lo + 1)).astype(np.int64)
    if exact32:
        m = (cls == 3) & (rng.random(n) < exact32)
        w[m] = 32
    return w.astype(np.int64)


def width_class(w):
    w = np.asarray(w)
    edges = np.array([1, 8, 16, 32, 64, 128, 512])
    return np.minimum(np.searchsorted(edges, w), NCLS - 1)


class _Pools:
    """Flat signal-id pools grouped by (group, class) for vectorised picking."""

    def __init__(self, groups: list[np.ndarray], widths: np.ndarray):
        self.ids = []
        self.off = np.zeros((len(groups), NCLS), np.int64)
        self.cnt = np.zeros((len(groups), NCLS), np.int64)
        pos = 0
        for g, sig in enumerate(groups):
            sig = np.asarray(sig, np.int64)
            cl = width_class(widths[sig]) if sig.size else np.zeros(0, np.int64)
            for c in range(NCLS):
                m = sig[cl == c]
                self.off[g, c] = pos
                self.cnt[g, c] = m.size
                self.ids.append(m)
                pos += m.size
        self.ids = np.concatenate(self.ids) if self.ids else np.zeros(0, np.int64)
        # fallback class: nearest non-empty class in the same group
        self.fb = np.zeros((len(groups), NCLS), np.int64)
        for g in range(len(groups)):
            ne = np.nonzero(self.cnt[g])[0]
            for c in range(NCLS):
                self.fb[g, c] = ne[np.argmin(np.abs(ne - c))] if ne.size else -1

    def pick(self, rng, g, c):
        """Vectorised: one random signal of class c (or the nearest class) from group g."""
        g = np.asarray(g, np.int64)
        c = self.fb[g, np.asarray(c, np.int64)]
        ok = c >= 0
        out = np.full(g.shape, -1, np.int64)
        if ok.any():
            gg, cc = g[ok], c[ok]
            idx = self.off[gg, cc] + (rng.random(gg.size) * self.cnt[gg, cc]).astype(np.int64)
            out[ok] = self.ids[idx]
        return out


def generate(config_id: int, seed: int | None = None, scale: float = 1.0) -> I.IR:
    """Generate the shaped design of ``config_id`` (2, 3 or 4).

    ``scale`` < 1 shrinks the op count (and registers) for fast tests while
    keeping every other shape parameter; the benchmark uses scale=1.
    Ops are emitted partition by partition, level by level, so the op order
    is topological (cross-partition operands come from earlier partitions).
    """
    sh = SHAPES[config_id]
    seed = DESIGN_SEED_BASE + config_id if seed is None else seed
    rng = np.random.default_rng(seed & ((1 << 63) - 1))
    n_ops = max(64, int(sh.n_ops * scale))
    P = sh.n_partitions if scale >= 1 else max(1, min(sh.n_partitions, int(round(sh.n_partitions * scale ** 0.5))))
    L = sh.levels_per_partition
    n_regs = max(40, int(n_ops * sh.reg_fraction))
    n_consts = max(8, int(n_ops * sh.const_fraction))

    cap = 1024 + n_ops + n_regs + n_consts + 512
    wbuf = np.zeros(cap, np.int64)
    kbuf = np.zeros(cap, np.int64)
    nsig = [0]

    def new_sigs(w, kind):
        w = np.array(w, np.int64).reshape(-1)
        s0 = nsig[0]
        wbuf[s0:s0 + w.size] = w
        kbuf[s0:s0 + w.size] = kind
        nsig[0] += w.size
        return np.arange(s0, s0 + w.size, dtype=np.int64)

    def W():
        return wbuf          # entries beyond nsig are never indexed

    # ---- inputs
    if sh.input_widths:
        in_w = np.asarray(sh.input_widths, np.int64)
    else:
        in_w = _sample_widths(rng, _N_INPUTS[config_id], sh.width_dist)
    inputs = new_sigs(in_w, I.INPUT)
    # ---- constants (values drawn at the end)
    c_w = _sample_widths(rng, n_consts, sh.width_dist, sh.exact32)
    c_w[: min(16, n_consts)] = rng.integers(2, 6, size=min(16, n_consts))   # shift amounts
    consts = list(new_sigs(c_w, I.CONST))
    const_vals: dict[int, int] = {}
    # ---- registers, owned by partitions in contiguous blocks
    r_w = _sample_widths(rng, n_regs, sh.width_dist, sh.exact32)
    if sh.regbank:
        r_w[:32] = 32
    regs = new_sigs(r_w, I.REG)
    reg_part = (np.arange(n_regs) * P) // n_regs
    reg_d = np.full(n_regs, -1, np.int64)

    op_names = np.array(list(OP_MIX))
    op_p = np.array([OP_MIX[k] for k in op_names], float)
    op_p /= op_p.sum()
    op_codes = np.array([I.OPCODES[k] for k in op_names], np.int64)
    unary = np.isin(op_names, list(I.UNARY))

    ops_list = []
    part_level = np.arange(P) // max(1, sh.partition_width)
    per_part = np.full(P, n_ops // P)
    per_part[: n_ops - per_part.sum()] += 1
    part_comb: list[np.ndarray] = []

    for p in range(P):
        wcur = W()
        reg_pool = _Pools([regs[reg_part == p], regs], wcur)   # 0 = own, 1 = any
        in_pool = _Pools([inputs], wcur)
        const_pool = _Pools([np.asarray(consts)], wcur)
        earlier = [q for q in range(P) if part_level[q] < part_level[p]]
        x_pool = _Pools([part_comb[q] for q in earlier], wcur) if earlier else None
        budget = int(per_part[p])
        bank_read = np.zeros(0, np.int64)
        if sh.regbank and p == 0:
            rows, bank_read = _regbank_read(new_sigs, regs[:32], inputs, p)
            ops_list.append(rows)
            budget -= rows.shape[0] + 32 * 3 + 1      # read trees + write decoders
        level_sizes = np.full(L, budget // L)
        level_sizes[: budget - level_sizes.sum()] += 1
        level_sigs: list[np.ndarray] = []
        level_pool = None
        for l in range(L):
            n = int(level_sizes[l])
            if n <= 0:
                continue
            opc_idx = rng.choice(op_codes.size, size=n, p=op_p)
            nm = op_names[opc_idx]
            opc = op_codes[opc_idx].copy()
            wd = _sample_widths(rng, n, sh.width_dist, sh.exact32)

            def operand(desired_cls):
                """Pick n operands with the SURVEY's source mix and locality."""
                u = rng.random(n)
                src = np.full(n, 4)                     # 4 = local comb
                acc = 0.0
                for code, pr in ((0, sh.p_reg), (1, sh.p_in), (2, sh.p_const),
                                 (3, sh.p_xpart if x_pool is not None else 0.0)):
                    src[(u >= acc) & (u < acc + pr)] = code
                    acc += pr
                if level_pool is None:
                    src[src == 4] = 0
                c = np.where(rng.random(n) < sh.same_class, desired_cls,
                             width_class(_sample_widths(rng, n, sh.width_dist, sh.exact32)))
                out = np.full(n, -1, np.int64)
                m = src == 0
                if m.any():
                    other = (rng.random(m.sum()) >= 0.95).astype(np.int64)
                    out[m] = reg_pool.pick(rng, other, c[m])
                m = src == 1
                if m.any():
                    out[m] = in_pool.pick(rng, np.zeros(m.sum(), np.int64), c[m])
                m = src == 2
                if m.any():
                    out[m] = const_pool.pick(rng, np.zeros(m.sum(), np.int64), c[m])
                m = src == 3
                if m.any():
                    g = rng.integers(0, len(earlier), size=m.sum())
                    out[m] = x_pool.pick(rng, g, c[m])
                m = src == 4
                if m.any():
                    nl = len(level_sigs)
                    back = rng.choice(len(sh.back_probs), size=m.sum(), p=sh.back_probs) + 1
                    back = np.minimum(back, nl)
                    out[m] = level_pool.pick(rng, nl - back, c[m])
                bad = out < 0
                if bad.any():
                    out[bad] = reg_pool.pick(rng, np.ones(bad.sum(), np.int64), c[bad])
                return out

            cls_d = width_class(wd)
            a = operand(cls_d)
            b = operand(cls_d)
            cc = operand(cls_d)
            imm = np.zeros(n, np.int64)
            wall = W()
            # ---- per-opcode operand / width rules
            wd[np.isin(nm, list(I.COMPARES | I.REDUCTIONS))] = 1
            md = np.isin(nm, list(I.MULDIV))
            if md.any():
                wd[md] = np.minimum(wd[md], 64)
                c64 = np.minimum(width_class(wd), 4)
                for _ in range(4):
                    bad = md & ((wall[a] > 64) | (wall[b] > 64))
                    if not bad.any():
                        break
                    a2, b2 = operand(c64), operand(c64)
                    a[bad], b[bad] = a2[bad], b2[bad]
                bad = md & ((wall[a] > 64) | (wall[b] > 64))
                nm[bad] = "AND"
                opc[bad] = I.OPCODES["AND"]
            sht = np.isin(nm, list(I.SHIFTS))
            if sht.any():
                b[sht] = operand(np.full(n, 1))[sht]          # 2-8 bit shift amounts
            mux = nm == "MUX"
            if mux.any():
                a[mux] = operand(np.zeros(n, np.int64))[mux]  # 1-bit selects
            wa, wb = wall[a], wall[b]
            sl = nm == "SLICE"
            if sl.any():
                wd[sl] = np.minimum(wd[sl], wa[sl])
                imm[sl] = (rng.random(sl.sum()) * (wa[sl] - wd[sl] + 1)).astype(np.int64)
            opc[(nm == "SEXT") & (wa > wd)] = I.OPCODES["COPY"]
            cat = nm == "CONCAT"
            wd[cat] = np.minimum(wa[cat] + wb[cat], I.MAX_WIDTH)
            dst = new_sigs(wd, I.COMB)
            is_unary = unary[opc_idx]
            bcol = np.where(is_unary, I.NONE, b)
            ccol = np.where(mux, cc, I.NONE)
            ops_list.append(np.stack([opc, np.full(n, p), dst, a, bcol, ccol, imm], axis=1))
            if l == min(6, L - 1) and bank_read.size:
                dst = np.concatenate([dst, bank_read])
            level_sigs.append(dst)
            level_pool = _Pools(level_sigs, W())
        part_comb.append(np.concatenate(level_sigs))
        # ---- register D from this partition's last levels (class-matched)
        mine = np.nonzero(reg_part == p)[0]
        if mine.size:
            last = _Pools([np.concatenate(level_sigs[-4:])], W())
            reg_d[mine] = last.pick(rng, np.zeros(mine.size, np.int64), width_class(r_w[mine]))
            if sh.regbank and p == 0:
                rows, d_bank, cs = _regbank_write(rng, new_sigs, regs[:32], level_sigs, W(), p)
                ops_list.append(rows)
                reg_d[:32] = d_bank
                for s_, v_ in cs:
                    consts.append(s_)
                    const_vals[s_] = v_
    # ---- outputs: comb values from the last levels of (spread) partitions
    wall = W()
    outs = []
    for j in range(sh.n_outputs):
        p = (j * P) // sh.n_outputs
        cand = part_comb[p][-max(2, 2 * (per_part[p] // L)):]
        narrow = cand[wall[cand] <= 64]
        cand = narrow if narrow.size else cand
        outs.append(int(cand[int(rng.integers(0, cand.size))]))
    width = wbuf[:nsig[0]].copy()
    kind = kbuf[:nsig[0]].copy()
    ops_arr = np.concatenate(ops_list, axis=0)
    ops = np.zeros(ops_arr.shape[0], dtype=I.OP_DTYPE)
    for k, f in enumerate(("opcode", "part", "dst", "a", "b", "c", "imm")):
        ops[f] = ops_arr[:, k]
    reg_init = []
    for q in regs:
        reg_init += I.int_to_words(0, int(width[q]))
    const_words = []
    for s in consts:
        w = int(width[s])
        v = const_vals.get(s)
        if v is None:
            v = int.from_bytes(rng.bytes((w + 7) // 8), "little") & ((1 << w) - 1)
        const_words += I.int_to_words(v, w)
    out = I.IR(width=width, kind=kind, ops=ops, reg_q=regs, reg_d=reg_d,
               reg_init=np.asarray(reg_init, np.uint32), const_sig=np.asarray(consts),
               const_words=np.asarray(const_words, np.uint32), input_sig=inputs,
               output_sig=np.asarray(outs), n_partitions=P,
               name=sh.name if scale >= 1 else f"{sh.name}@{scale:g}")
    out.meta = {"config_id": config_id, "seed": seed, "scale": scale}
    return out


def _regbank_read(new_sigs, bank, inputs, p):
    """32 x 32-bit register bank (riscv-mini register file shape): two 32:1
    read mux trees addressed by 5-bit slices of the two 32-bit inputs."""
    rows = []
    outs = []
    for port in range(2):
        addr_src = int(inputs[port])
        bits = []
        for k in range(5):
            s = int(new_sigs([1], I.COMB)[0])
            rows.append([I.OPCODES["SLICE"], p, s, addr_src, I.NONE, I.NONE, 15 + 5 * port + k])
            bits.append(s)
        layer = [int(x) for x in bank]
        for k in range(5):
            nxt = []
            for j in range(0, len(layer), 2):
                s = int(new_sigs([32], I.COMB)[0])
                rows.append([I.OPCODES["MUX"], p, s, bits[k], layer[j + 1], layer[j], 0])
                nxt.append(s)
            layer = nxt
        outs.append(layer[0])
    return np.asarray(rows, np.int64), np.asarray(outs, np.int64)


def _regbank_write(rng, new_sigs, bank, level_sigs, wall, p):
    """Decoded write enables: we_i = (waddr == i) & wen; d_i = we_i ? wdata : q_i."""
    late = np.concatenate(level_sigs[-4:-2])
    w32 = late[wall[late] == 32]
    w1 = late[wall[late] == 1]
    wdata = int(w32[int(rng.integers(0, w32.size))]) if w32.size else int(late[0])
    wen = int(w1[int(rng.integers(0, w1.size))]) if w1.size else int(late[0])
    rows = []
    consts = []
    waddr = int(new_sigs([5], I.COMB)[0])
    rows.append([I.OPCODES["SLICE"], p, waddr, wdata, I.NONE, I.NONE, 0])
    d = np.zeros(len(bank), np.int64)
    for i, q in enumerate(bank):
        ci = int(new_sigs([5], I.CONST)[0])
        consts.append((ci, i))
        eq = int(new_sigs([1], I.COMB)[0])
        rows.append([I.OPCODES["EQ"], p, eq, waddr, ci, I.NONE, 0])
        we = int(new_sigs([1], I.COMB)[0])
        rows.append([I.OPCODES["AND"], p, we, eq, wen, I.NONE, 0])
        dn = int(new_sigs([32], I.COMB)[0])
        rows.append([I.OPCODES["MUX"], p, dn, we, wdata, int(q), 0])
        d[i] = dn
    return np.asarray(rows, np.int64), d, consts
