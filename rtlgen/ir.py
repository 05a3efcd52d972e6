"""Levelized RTL IR container — the interchange format both sides consume.

This module is INPUT PLUMBING shared by the oracle tests and the CUDA path
(the only kind of code the two may share): it defines the IR's field layout
and opcode numbering (an interface, mirrored in ``include/rtlsim.h`` and,
independently, in ``oracle/oracle.h``) and holds NO simulation arithmetic.

The IR is the compact stand-in for the RTL graph of PAPER.md §2 (P:L201-207:
"nodes represent logic elements ... edges represent wires") after the
Verilator front end, which is out of scope.
Operation semantics are specified in DESIGN.md §3.
"""
from __future__ import annotations

import dataclasses
import numpy as np

# ---------------------------------------------------------------- opcodes --
# Numbering is part of the interface (rtlsim.h enum rtlsim_opcode).
OPCODES = {
    "COPY": 0,    # zero-extend / truncate
    "SEXT": 1,
    "NOT": 2,
    "AND": 3,
    "OR": 4,
    "XOR": 5,
    "ADD": 6,
    "SUB": 7,
    "NEG": 8,
    "MUL": 9,
    "DIVU": 10,
    "MODU": 11,
    "EQ": 12,
    "NE": 13,
    "LTU": 14,
    "LEU": 15,
    "GTU": 16,
    "GEU": 17,
    "LTS": 18,
    "LES": 19,
    "GTS": 20,
    "GES": 21,
    "SHL": 22,
    "SHRL": 23,
    "SHRA": 24,
    "MUX": 25,    # a = select, b = then, c = else
    "CONCAT": 26,  # {a, b}: a is the high part
    "SLICE": 27,  # a[imm + wd - 1 : imm]
    "REDAND": 28,
    "REDOR": 29,
    "REDXOR": 30,
    "MEMRD": 31,  # dst := MEM[imm][a] (0 when a >= depth): ARRSEL read (reading 12)
}
OPNAMES = {v: k for k, v in OPCODES.items()}
MEM_OPS = {"MEMRD"}                       # reads a memory: not a function of its operands alone
VALUE_OPS = [k for k in OPCODES if k not in MEM_OPS]
N_OPCODES = len(OPCODES)
globals().update({"OP_" + k: v for k, v in OPCODES.items()})

UNARY = {"COPY", "SEXT", "NOT", "NEG", "REDAND", "REDOR", "REDXOR", "SLICE", "MEMRD"}
TERNARY = {"MUX"}
COMPARES = {"EQ", "NE", "LTU", "LEU", "GTU", "GEU", "LTS", "LES", "GTS", "GES"}
REDUCTIONS = {"REDAND", "REDOR", "REDXOR"}
MULDIV = {"MUL", "DIVU", "MODU"}
SHIFTS = {"SHL", "SHRL", "SHRA"}

# signal kinds
INPUT, REG, COMB, CONST = 0, 1, 2, 3
NONE = 0xFFFFFFFF
MAX_WIDTH = 1024
MAX_MULDIV_WIDTH = 64

OP_DTYPE = np.dtype([
    ("opcode", "<u2"), ("part", "<u2"),
    ("dst", "<u4"), ("a", "<u4"), ("b", "<u4"), ("c", "<u4"), ("imm", "<u4"),
])
assert OP_DTYPE.itemsize == 24


def nwords(w) -> int | np.ndarray:
    """Number of little-endian u32 words that hold a w-bit value."""
    return (np.asarray(w, dtype=np.int64) + 31) // 32 if isinstance(w, np.ndarray) else (int(w) + 31) // 32


def int_to_words(v: int, w: int) -> list[int]:
    v &= (1 << w) - 1
    return [(v >> (32 * i)) & 0xFFFFFFFF for i in range(nwords(w))]


def words_to_int(ws) -> int:
    return sum(int(x) << (32 * i) for i, x in enumerate(ws))


@dataclasses.dataclass
class IR:
    """A levelized design. Arrays mirror ``rtlsim_ir`` field for field."""
    width: np.ndarray          # u16 [n_signals], 1..1024
    kind: np.ndarray           # u8  [n_signals]
    ops: np.ndarray            # OP_DTYPE [n_ops], topological order
    reg_q: np.ndarray          # u32 [n_regs]
    reg_d: np.ndarray          # u32 [n_regs]
    reg_init: np.ndarray       # u32 [sum ceil(w_q/32)]
    const_sig: np.ndarray      # u32 [n_consts]
    const_words: np.ndarray    # u32 [sum ceil(w/32)]
    input_sig: np.ndarray      # u32 [n_inputs]
    output_sig: np.ndarray     # u32 [n_outputs]
    n_partitions: int = 1
    name: str = "design"
    meta: dict = dataclasses.field(default_factory=dict)
    # memories (ARRSEL, §3.1.1 Fig 5; reading 12): memory m
    # has mem_depth[m] entries of mem_width[m] bits; mem_init holds every
    # entry's words (memory-major, entry-major); write port p is
    # mem_wport[p] = (mem, addr signal, data signal, enable signal)
    mem_width: np.ndarray = dataclasses.field(default_factory=lambda: np.zeros(0, np.uint16))
    mem_depth: np.ndarray = dataclasses.field(default_factory=lambda: np.zeros(0, np.uint32))
    mem_init: np.ndarray = dataclasses.field(default_factory=lambda: np.zeros(0, np.uint32))
    mem_wport: np.ndarray = dataclasses.field(default_factory=lambda: np.zeros((0, 4), np.uint32))

    def __post_init__(self):
        self.width = np.ascontiguousarray(self.width, dtype=np.uint16)
        self.kind = np.ascontiguousarray(self.kind, dtype=np.uint8)
        self.ops = np.ascontiguousarray(self.ops, dtype=OP_DTYPE)
        for f in ("reg_q", "reg_d", "reg_init", "const_sig", "const_words", "input_sig", "output_sig",
                  "mem_depth", "mem_init"):
            setattr(self, f, np.ascontiguousarray(getattr(self, f), dtype=np.uint32))
        self.mem_width = np.ascontiguousarray(self.mem_width, dtype=np.uint16)
        self.mem_wport = np.ascontiguousarray(self.mem_wport, dtype=np.uint32).reshape(-1, 4)

    # ------------------------------------------------------------ sizes --
    @property
    def n_signals(self) -> int:
        return int(self.width.shape[0])

    @property
    def n_ops(self) -> int:
        return int(self.ops.shape[0])

    @property
    def n_regs(self) -> int:
        return int(self.reg_q.shape[0])

    def _words(self, sigs) -> int:
        if len(sigs) == 0:
            return 0
        return int(nwords(self.width[np.asarray(sigs, dtype=np.int64)].astype(np.int64)).sum())

    @property
    def IW(self) -> int:
        return self._words(self.input_sig)

    @property
    def OW(self) -> int:
        return self._words(self.output_sig)

    @property
    def RW(self) -> int:
        return self._words(self.reg_q)

    @property
    def n_mems(self) -> int:
        return int(self.mem_width.shape[0])

    @property
    def MW(self) -> int:
        """words of all memories of one stimulus"""
        if not self.n_mems:
            return 0
        return int((nwords(self.mem_width.astype(np.int64)) * self.mem_depth.astype(np.int64)).sum())

    def input_word_masks(self) -> np.ndarray:
        """u32 mask per stimulus word (bits >= width are ignored, reading 15)."""
        out = []
        for s in self.input_sig:
            w = int(self.width[s])
            for i in range(nwords(w)):
                bits = min(32, w - 32 * i)
                out.append((1 << bits) - 1)
        return np.asarray(out, dtype=np.uint32)

    # --------------------------------------------------------- file I/O --
    def save(self, path: str) -> None:
        np.savez_compressed(
            path, width=self.width, kind=self.kind, ops=self.ops.view(np.uint8),
            reg_q=self.reg_q, reg_d=self.reg_d, reg_init=self.reg_init,
            const_sig=self.const_sig, const_words=self.const_words,
            input_sig=self.input_sig, output_sig=self.output_sig,
            n_partitions=np.asarray(self.n_partitions), name=np.asarray(self.name),
            mem_width=self.mem_width, mem_depth=self.mem_depth, mem_init=self.mem_init,
            mem_wport=self.mem_wport)

    @classmethod
    def load(cls, path: str) -> "IR":
        z = np.load(path)
        return cls(width=z["width"], kind=z["kind"], ops=z["ops"].view(OP_DTYPE),
                   reg_q=z["reg_q"], reg_d=z["reg_d"], reg_init=z["reg_init"],
                   const_sig=z["const_sig"], const_words=z["const_words"],
                   input_sig=z["input_sig"], output_sig=z["output_sig"],
                   n_partitions=int(z["n_partitions"]), name=str(z["name"]),
                   **{k: z[k] for k in ("mem_width", "mem_depth", "mem_init", "mem_wport") if k in z})

    def summary(self) -> dict:
        ops = self.ops
        hist = np.bincount(ops["opcode"], minlength=N_OPCODES) if self.n_ops else np.zeros(N_OPCODES, int)
        return {
            "name": self.name, "n_signals": self.n_signals, "n_ops": self.n_ops,
            "n_regs": self.n_regs, "n_inputs": int(self.input_sig.size),
            "n_outputs": int(self.output_sig.size), "IW": self.IW, "OW": self.OW,
            "RW": self.RW, "n_partitions": self.n_partitions,
            "opcode_hist": {OPNAMES[i]: int(h) for i, h in enumerate(hist) if h},
        }
