"""CPU oracle for the levelized RTL IR — TEST INFRASTRUCTURE ONLY.

Only ``tests/``, ``__graft_entry__.smoke()`` and ``bench.py``'s
``cpu_baseline`` / ``--impl reference`` leg may import this package. The
product package (``paper_conf_icpp_linrzkh22_b200``) never imports it.

* :mod:`oracle.ops_ref` — per-op mathematical definitions on Python ints.
* :mod:`oracle.pysim`   — a pure-Python cycle loop over ``ops_ref`` (small cases).
* :func:`simulate`      — the plain C interpreter ``liboracle.so`` (oracle.c),
  single- or multi-threaded over stimuli.

Algorithm: PAPER.md Listing 1 with the readings of DESIGN.md §3.
"""
from __future__ import annotations

import ctypes
import os
import subprocess

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "liboracle.so")
_lib = None


def build(force: bool = False) -> str:
    """Compile oracle.c with gcc (plain -O2; loops are not turned into memset calls, whose start-up cost dominated the small per-op scratch clears)."""
    src = os.path.join(_HERE, "oracle.c")
    if force or not os.path.exists(LIB_PATH) or os.path.getmtime(LIB_PATH) < max(
            os.path.getmtime(src), os.path.getmtime(os.path.join(_HERE, "oracle.h"))):
        subprocess.check_call(["gcc", "-O2", "-fno-tree-loop-distribute-patterns", "-std=c11", "-Wall", "-shared", "-fPIC", "-pthread",
                               "-o", LIB_PATH, src])
    return LIB_PATH


class _Op(ctypes.Structure):
    _fields_ = [("opcode", ctypes.c_uint16), ("part", ctypes.c_uint16), ("dst", ctypes.c_uint32),
                ("a", ctypes.c_uint32), ("b", ctypes.c_uint32), ("c", ctypes.c_uint32),
                ("imm", ctypes.c_uint32)]


def lib():
    global _lib
    if _lib is None:
        build()
        L = ctypes.CDLL(LIB_PATH)
        P = ctypes.c_void_p
        u32, u64 = ctypes.c_uint32, ctypes.c_uint64
        L.oracle_design_new.restype = P
        L.oracle_design_new.argtypes = [u32, P, P, u32, P, u32, P, P, P, u32, P, P, u32, P, u32, P,
                                        ctypes.c_char_p, ctypes.c_int]
        L.oracle_design_free.argtypes = [P]
        L.oracle_simulate.restype = ctypes.c_int
        L.oracle_simulate.argtypes = [P, u64, u64, P, P, P, P, P, ctypes.c_int, ctypes.c_char_p, ctypes.c_int]
        L.oracle_eval_op.restype = ctypes.c_int
        L.oracle_eval_op.argtypes = [u32, u32, u32, P, u32, P, u32, P, u32, P]
        L.oracle_mix64.restype = u64
        L.oracle_mix64.argtypes = [u64]
        for f in ("oracle_iw", "oracle_ow", "oracle_rw"):
            getattr(L, f).restype = u32
            getattr(L, f).argtypes = [P]
        L.oracle_design_set_mems.restype = ctypes.c_int
        L.oracle_design_set_mems.argtypes = [P, u32, P, P, P, u32, P, ctypes.c_char_p, ctypes.c_int]
        L.oracle_mw.restype = u64
        L.oracle_mw.argtypes = [P]
        L.oracle_simulate_mem.restype = ctypes.c_int
        L.oracle_simulate_mem.argtypes = [P, u64, u64, P, P, P, P, P, P, ctypes.c_int, ctypes.c_char_p,
                                          ctypes.c_int]
        _lib = L
    return _lib


def _p(a):
    return None if a is None else a.ctypes.data_as(ctypes.c_void_p)


class Design:
    """An IR loaded into the C oracle."""

    def __init__(self, ir):
        L = lib()
        self.ir = ir
        err = ctypes.create_string_buffer(256)
        self._keep = [ir.width, ir.kind, ir.ops, ir.reg_q, ir.reg_d, ir.reg_init, ir.const_sig,
                      ir.const_words, ir.input_sig, ir.output_sig]
        h = L.oracle_design_new(ir.n_signals, _p(ir.width), _p(ir.kind), ir.n_ops, _p(ir.ops),
                                ir.n_regs, _p(ir.reg_q), _p(ir.reg_d), _p(ir.reg_init),
                                int(ir.const_sig.size), _p(ir.const_sig), _p(ir.const_words),
                                int(ir.input_sig.size), _p(ir.input_sig),
                                int(ir.output_sig.size), _p(ir.output_sig), err, 256)
        if not h:
            raise ValueError("oracle rejected IR: " + err.value.decode())
        self.h = h
        self.IW, self.OW, self.RW = L.oracle_iw(h), L.oracle_ow(h), L.oracle_rw(h)
        if getattr(ir, "n_mems", 0) or getattr(ir, "mem_wport", np.zeros((0, 4))).size:
            self._keep += [ir.mem_width, ir.mem_depth, ir.mem_init, ir.mem_wport]
            rc = L.oracle_design_set_mems(h, ir.n_mems, _p(ir.mem_width), _p(ir.mem_depth), _p(ir.mem_init),
                                          int(ir.mem_wport.shape[0]), _p(ir.mem_wport), err, 256)
            if rc:
                raise ValueError("oracle rejected memories: " + err.value.decode())
        self.MW = int(L.oracle_mw(h))

    def __del__(self):
        if getattr(self, "h", None):
            lib().oracle_design_free(self.h)
            self.h = None

    def simulate(self, stim, regs_in=None, out=True, regs=True, digest=False, threads=1, mems=False):
        """stim [N][T][IW] u32 -> dict(out [N][T][OW], regs [N][RW], digest [N][T],
        mems [N][MW] final memory words when mems=True)."""
        stim = np.ascontiguousarray(stim, dtype=np.uint32)
        N, T = int(stim.shape[0]), int(stim.shape[1])
        assert stim.shape[2] == self.IW, (stim.shape, self.IW)
        o = np.zeros((N, T, self.OW), np.uint32) if out else None
        r = np.zeros((N, self.RW), np.uint32) if regs else None
        dg = np.zeros((N, T), np.uint64) if digest else None
        rin = None if regs_in is None else np.ascontiguousarray(regs_in, dtype=np.uint32)
        m = np.zeros((N, self.MW), np.uint32) if mems and self.MW else None
        err = ctypes.create_string_buffer(256)
        rc = lib().oracle_simulate_mem(self.h, N, T, _p(stim), _p(rin), _p(o), _p(r), _p(dg), _p(m),
                                       int(threads), err, 256)
        if rc:
            raise RuntimeError(err.value.decode())
        return {"out": o, "regs": r, "digest": dg, "mems": m}


def simulate(ir, stim, **kw):
    return Design(ir).simulate(stim, **kw)


def eval_op(opcode: int, wd: int, a: int, wa: int, b: int = 0, wb: int = 0, c: int = 0,
            wc: int = 0, imm: int = 0) -> int:
    """One op on Python-int operands through the C oracle's EVAL."""
    from rtlgen.ir import int_to_words, words_to_int, nwords
    A = np.asarray(int_to_words(a, wa), np.uint32)
    B = np.asarray(int_to_words(b, max(wb, 1)), np.uint32)
    C = np.asarray(int_to_words(c, max(wc, 1)), np.uint32)
    R = np.zeros(nwords(wd), np.uint32)
    rc = lib().oracle_eval_op(opcode, wd, imm, _p(A), wa, _p(B) if wb else None, wb,
                              _p(C) if wc else None, wc, _p(R))
    if rc:
        raise ValueError("unsupported")
    return words_to_int(R)


def mix64(z: int) -> int:
    return int(lib().oracle_mix64(z & ((1 << 64) - 1)))
