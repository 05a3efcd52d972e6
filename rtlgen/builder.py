"""Incremental builder for hand-written IR designs (tiny DUTs, test fixtures).

Input plumbing only: it records signals and ops; it evaluates nothing.
"""
from __future__ import annotations

import numpy as np

from . import ir as I


class Builder:
    def __init__(self, name: str = "design"):
        self.name = name
        self.width: list[int] = []
        self.kind: list[int] = []
        self.ops: list[tuple] = []
        self.regs: list[list] = []          # [q, d, init]
        self.consts: list[tuple[int, int]] = []   # (sig, value)
        self.inputs: list[int] = []
        self.outputs: list[int] = []
        self.names: dict[int, str] = {}
        self.part = 0
        self.n_partitions = 1
        self.mems: list[tuple[int, int, list[int]]] = []   # (width, depth, init values)
        self.wports: list[tuple[int, int, int, int]] = []  # (mem, addr, data, en)

    # ---------------------------------------------------------- signals --
    def _sig(self, w: int, kind: int, name: str | None) -> int:
        s = len(self.width)
        self.width.append(int(w))
        self.kind.append(kind)
        if name:
            self.names[s] = name
        return s

    def input(self, w: int, name: str | None = None) -> int:
        s = self._sig(w, I.INPUT, name)
        self.inputs.append(s)
        return s

    def reg(self, w: int, init: int = 0, name: str | None = None) -> int:
        s = self._sig(w, I.REG, name)
        self.regs.append([s, None, int(init)])
        return s

    def const(self, w: int, value: int, name: str | None = None) -> int:
        s = self._sig(w, I.CONST, name)
        self.consts.append((s, int(value)))
        return s

    def set_d(self, q: int, d: int) -> None:
        for r in self.regs:
            if r[0] == q:
                r[1] = d
                return
        raise KeyError(q)

    def output(self, sig: int) -> int:
        self.outputs.append(sig)
        return sig

    def partition(self, p: int) -> None:
        self.part = p
        self.n_partitions = max(self.n_partitions, p + 1)

    # -------------------------------------------------------------- ops --
    def op(self, name: str, w: int, a: int, b: int | None = None, c: int | None = None,
           imm: int = 0, out_name: str | None = None) -> int:
        d = self._sig(w, I.COMB, out_name)
        self.ops.append((I.OPCODES[name], self.part, d,
                         I.NONE if a is None else a,
                         I.NONE if b is None else b,
                         I.NONE if c is None else c, imm))
        return d

    def __getattr__(self, item):
        # b.ADD(w, a, b) sugar
        if item.isupper() and item in I.OPCODES:
            return lambda w, *args, **kw: self.op(item, w, *args, **kw)
        raise AttributeError(item)

    def slice(self, a: int, lo: int, w: int) -> int:
        return self.op("SLICE", w, a, imm=lo)

    # --------------------------------------------------------- memories --
    def mem(self, width: int, depth: int, init=None) -> int:
        """A memory of `depth` entries of `width` bits (ARRSEL target)."""
        init = [0] * depth if init is None else [int(v) for v in init]
        assert len(init) == depth
        self.mems.append((int(width), int(depth), init))
        return len(self.mems) - 1

    def memrd(self, m: int, addr: int, out_name: str | None = None) -> int:
        """Combinational read of entry `addr` of memory m (MEMRD)."""
        return self.op("MEMRD", self.mems[m][0], addr, imm=m, out_name=out_name)

    def wport(self, m: int, addr: int, data: int, en: int) -> None:
        """Synchronous write port: at the clock edge, if en: mem[addr] := data."""
        self.wports.append((m, addr, data, en))

    # ------------------------------------------------------------ build --
    def build(self) -> I.IR:
        for q, d, _ in self.regs:
            if d is None:
                raise ValueError(f"register {self.names.get(q, q)} has no D")
        width = np.asarray(self.width, dtype=np.uint16)
        ops = np.zeros(len(self.ops), dtype=I.OP_DTYPE)
        for i, t in enumerate(self.ops):
            ops[i] = t
        reg_init = []
        for q, _, init in self.regs:
            reg_init += I.int_to_words(init, int(width[q]))
        const_words = []
        for s, v in self.consts:
            const_words += I.int_to_words(v, int(width[s]))
        return I.IR(
            width=width, kind=np.asarray(self.kind, dtype=np.uint8), ops=ops,
            reg_q=[r[0] for r in self.regs], reg_d=[r[1] for r in self.regs],
            reg_init=np.asarray(reg_init, dtype=np.uint32),
            const_sig=[c[0] for c in self.consts],
            const_words=np.asarray(const_words, dtype=np.uint32),
            input_sig=self.inputs, output_sig=self.outputs,
            n_partitions=self.n_partitions, name=self.name,
            meta={"names": dict(self.names)},
            mem_width=np.asarray([m[0] for m in self.mems], dtype=np.uint16),
            mem_depth=np.asarray([m[1] for m in self.mems], dtype=np.uint32),
            mem_init=np.asarray([w for m in self.mems for v in m[2] for w in I.int_to_words(v, m[0])],
                                dtype=np.uint32),
            mem_wport=np.asarray(self.wports, dtype=np.uint32).reshape(-1, 4))
