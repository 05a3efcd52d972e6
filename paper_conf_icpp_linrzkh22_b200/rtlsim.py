"""Thin ctypes binding of the C ABI in include/rtlsim.h (argument marshalling only).

Every step of the simulation runs in librtlsim.so's CUDA kernels; this module
only converts numpy arrays / torch tensors to pointers. It never falls back to
any CPU implementation: if the shared library is missing or the device is
unavailable the calls raise.

Module-level functions carry the C names (``rtlsim_load``, ``rtlsim_bind``,
``rtlsim_run`` ...); :class:`Simulator` is a small convenience wrapper.
"""
from __future__ import annotations

import ctypes
import os

import numpy as np

_HERE = os.path.dirname(os.path.abspath(__file__))
LIB_PATH = os.path.join(_HERE, "librtlsim.so")

RTLSIM_OK = 0
STATUS = {0: "OK", -1: "E_ARG", -2: "E_IR", -3: "E_COMB_LOOP", -4: "E_UNSUPPORTED", -5: "E_NOMEM",
          -6: "E_CUDA", -7: "E_STATE", -8: "E_RANGE"}
F_DIGEST, F_NO_PIPELINE, F_GRAPH, F_HOST_ONLY, F_TIMING, F_JIT, F_V4, F_STREAM = 0x1, 0x2, 0x4, 0x8, 0x10, 0x20, 0x40, 0x80
# F_V4 is reserved (the removed run-based evaluator): loading with it fails with E_UNSUPPORTED
F_NO_DCE = 0x100
F_COVERAGE = 0x200

EXPORTS = ["rtlsim_load", "rtlsim_bind", "rtlsim_bind_device", "rtlsim_bind_stream", "rtlsim_run",
           "rtlsim_run_device", "rtlsim_run_stream", "rtlsim_sync", "rtlsim_get_regs", "rtlsim_set_regs",
           "rtlsim_reset", "rtlsim_coverage", "rtlsim_reg_digest", "rtlsim_get_mems", "rtlsim_stats", "rtlsim_launch_count", "rtlsim_last_error", "rtlsim_free"]


class RtlsimError(RuntimeError):
    def __init__(self, code: int, msg: str):
        super().__init__(f"{STATUS.get(code, code)}: {msg}")
        self.code = code


class Op(ctypes.Structure):
    _fields_ = [("opcode", ctypes.c_uint16), ("part", ctypes.c_uint16), ("dst", ctypes.c_uint32),
                ("a", ctypes.c_uint32), ("b", ctypes.c_uint32), ("c", ctypes.c_uint32), ("imm", ctypes.c_uint32)]


_P = ctypes.c_void_p


class IRStruct(ctypes.Structure):
    _fields_ = [("n_signals", ctypes.c_uint32), ("width", _P), ("kind", _P),
                ("n_ops", ctypes.c_uint32), ("ops", _P),
                ("n_regs", ctypes.c_uint32), ("reg_q", _P), ("reg_d", _P), ("reg_init", _P),
                ("n_consts", ctypes.c_uint32), ("const_sig", _P), ("const_words", _P),
                ("n_inputs", ctypes.c_uint32), ("input_sig", _P),
                ("n_outputs", ctypes.c_uint32), ("output_sig", _P),
                ("n_partitions", ctypes.c_uint32),
                ("n_mems", ctypes.c_uint32), ("mem_width", _P), ("mem_depth", _P), ("mem_init", _P),
                ("n_wports", ctypes.c_uint32), ("mem_wport", _P)]


class Options(ctypes.Structure):
    _fields_ = [("device", ctypes.c_int), ("cuda_stream", _P), ("op_lanes", ctypes.c_uint32),
                ("chunk_cycles", ctypes.c_uint32), ("flags", ctypes.c_uint32), ("smem_limit", ctypes.c_uint32)]


class Stats(ctypes.Structure):
    _fields_ = [("n_ops", ctypes.c_uint64), ("n_signals", ctypes.c_uint64), ("n_regs", ctypes.c_uint64),
                ("word_ops", ctypes.c_uint64), ("n_desc", ctypes.c_uint64), ("n_steps", ctypes.c_uint64),
                ("n_partitions", ctypes.c_uint64), ("b_floor", ctypes.c_double), ("b_state", ctypes.c_double),
                ("b_part", ctypes.c_double),
                ("rows_bit", ctypes.c_uint64), ("rows_u8", ctypes.c_uint64), ("rows_u16", ctypes.c_uint64),
                ("rows_u32", ctypes.c_uint64), ("xrows_bit", ctypes.c_uint64), ("xrows_u8", ctypes.c_uint64),
                ("xrows_u16", ctypes.c_uint64), ("xrows_u32", ctypes.c_uint64), ("smem_words", ctypes.c_uint64),
                ("op_lanes", ctypes.c_uint32), ("chunk_cycles", ctypes.c_uint32), ("tile_stimuli", ctypes.c_uint32),
                ("iw", ctypes.c_uint32), ("ow", ctypes.c_uint32), ("rw", ctypes.c_uint32),
                ("device_bytes", ctypes.c_uint64), ("eval_ms", ctypes.c_double),
                ("eval_launches", ctypes.c_uint64), ("eval_stim_cycles", ctypes.c_uint64),
                ("jit_compile_s", ctypes.c_double), ("jit_cubin_bytes", ctypes.c_uint64),
                ("n_bitops", ctypes.c_uint64), ("n_narrow", ctypes.c_uint64), ("n_wide", ctypes.c_uint64),
                ("n_ld", ctypes.c_uint64), ("n_st", ctypes.c_uint64), ("b_spill", ctypes.c_double),
                ("n_live_ops", ctypes.c_uint64), ("live_word_ops", ctypes.c_uint64),
                ("jit_sass_instructions", ctypes.c_uint64), ("jit_tiles_per_cta", ctypes.c_uint32),
                ("tmem_cols", ctypes.c_uint32)]


PRODUCER = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64,
                            ctypes.POINTER(ctypes.c_uint32))
CONSUMER = ctypes.CFUNCTYPE(ctypes.c_int, ctypes.c_void_p, ctypes.c_uint64, ctypes.c_uint64,
                            ctypes.POINTER(ctypes.c_uint32), ctypes.POINTER(ctypes.c_uint64))

_lib = None


def lib():
    """Load librtlsim.so (raises if it was not built — there is no fallback)."""
    global _lib
    if _lib is None:
        if not os.path.exists(LIB_PATH):
            raise ImportError(f"{LIB_PATH} is missing: run __graft_entry__.build() "
                              "(python paper_conf_icpp_linrzkh22_b200/build.py)")
        L = ctypes.CDLL(LIB_PATH)
        u64, c_int = ctypes.c_uint64, ctypes.c_int
        L.rtlsim_load.argtypes = [ctypes.POINTER(IRStruct), ctypes.POINTER(Options), ctypes.POINTER(_P)]
        L.rtlsim_bind.argtypes = [_P, u64, u64, _P]
        L.rtlsim_bind_device.argtypes = [_P, u64, u64, _P]
        L.rtlsim_bind_stream.argtypes = [_P, u64, u64, PRODUCER, _P]
        L.rtlsim_run.argtypes = [_P, u64, _P, _P, _P]
        L.rtlsim_run_device.argtypes = [_P, u64, _P, _P]
        L.rtlsim_run_stream.argtypes = [_P, u64, CONSUMER, _P]
        L.rtlsim_sync.argtypes = [_P]
        L.rtlsim_get_regs.argtypes = [_P, _P]
        L.rtlsim_set_regs.argtypes = [_P, _P]
        L.rtlsim_reset.argtypes = [_P]
        L.rtlsim_coverage.argtypes = [_P, _P, c_int]
        L.rtlsim_reg_digest.argtypes = [_P, _P]
        L.rtlsim_get_mems.argtypes = [_P, _P]
        L.rtlsim_stats.argtypes = [_P, ctypes.POINTER(Stats)]
        L.rtlsim_launch_count.argtypes = [_P]
        L.rtlsim_launch_count.restype = u64
        L.rtlsim_last_error.argtypes = [_P]
        L.rtlsim_last_error.restype = ctypes.c_char_p
        L.rtlsim_free.argtypes = [_P]
        L.rtlsim_free.restype = None
        for f in EXPORTS:
            if f not in ("rtlsim_launch_count", "rtlsim_last_error", "rtlsim_free"):
                getattr(L, f).restype = c_int
        _lib = L
    return _lib


def _ptr(a):
    if a is None:
        return None
    if hasattr(a, "data_ptr"):          # torch tensor
        return ctypes.c_void_p(a.data_ptr())
    return a.ctypes.data_as(ctypes.c_void_p)


def _check(rc, ctx=None):
    if rc != RTLSIM_OK:
        msg = lib().rtlsim_last_error(ctx)
        raise RtlsimError(rc, msg.decode() if msg else "")


# ------------------------------------------------------- C-named wrappers --
def make_ir_struct(ir):
    """IRStruct pointing into the IR's numpy arrays (keep `ir` alive)."""
    s = IRStruct()
    s.n_signals = ir.width.size
    s.width, s.kind = _ptr(ir.width), _ptr(ir.kind)
    s.n_ops = ir.ops.size
    s.ops = _ptr(ir.ops)
    s.n_regs = ir.reg_q.size
    s.reg_q, s.reg_d, s.reg_init = _ptr(ir.reg_q), _ptr(ir.reg_d), _ptr(ir.reg_init)
    s.n_consts = ir.const_sig.size
    s.const_sig, s.const_words = _ptr(ir.const_sig), _ptr(ir.const_words)
    s.n_inputs = ir.input_sig.size
    s.input_sig = _ptr(ir.input_sig)
    s.n_outputs = ir.output_sig.size
    s.output_sig = _ptr(ir.output_sig)
    s.n_partitions = int(ir.n_partitions)
    n_mems = int(getattr(ir, "n_mems", 0))
    if n_mems or getattr(ir, "mem_wport", np.zeros((0, 4))).size:
        s.n_mems = n_mems
        s.mem_width, s.mem_depth, s.mem_init = _ptr(ir.mem_width), _ptr(ir.mem_depth), _ptr(ir.mem_init)
        s.n_wports = int(ir.mem_wport.shape[0])
        s.mem_wport = _ptr(ir.mem_wport)
    return s


def rtlsim_load(ir, device=0, stream=None, op_lanes=0, chunk_cycles=0, flags=0, smem_limit=0):
    s = make_ir_struct(ir)
    o = Options(device, stream, op_lanes, chunk_cycles, flags, smem_limit)
    h = _P()
    _check(lib().rtlsim_load(ctypes.byref(s), ctypes.byref(o), ctypes.byref(h)))
    return h


def rtlsim_bind(ctx, stim: np.ndarray):
    N, T = stim.shape[0], stim.shape[1]
    _check(lib().rtlsim_bind(ctx, N, T, _ptr(stim)), ctx)


def rtlsim_bind_device(ctx, stim_dev, N: int, T: int):
    _check(lib().rtlsim_bind_device(ctx, N, T, _ptr(stim_dev)), ctx)


def rtlsim_bind_stream(ctx, N: int, T: int, producer):
    _check(lib().rtlsim_bind_stream(ctx, N, T, producer, None), ctx)


def rtlsim_run(ctx, cycles: int, out=None, regs=None, digest=None):
    _check(lib().rtlsim_run(ctx, cycles, _ptr(out), _ptr(regs), _ptr(digest)), ctx)


def rtlsim_run_device(ctx, cycles: int, out_dev=None, digest_dev=None):
    _check(lib().rtlsim_run_device(ctx, cycles, _ptr(out_dev), _ptr(digest_dev)), ctx)


def rtlsim_run_stream(ctx, cycles: int, consumer):
    _check(lib().rtlsim_run_stream(ctx, cycles, consumer, None), ctx)


def rtlsim_sync(ctx):
    _check(lib().rtlsim_sync(ctx), ctx)


def rtlsim_get_regs(ctx, regs):
    _check(lib().rtlsim_get_regs(ctx, _ptr(regs)), ctx)


def rtlsim_set_regs(ctx, regs):
    _check(lib().rtlsim_set_regs(ctx, _ptr(regs)), ctx)


def rtlsim_reset(ctx):
    _check(lib().rtlsim_reset(ctx), ctx)


def rtlsim_coverage(ctx, bitmap, clear=False):
    _check(lib().rtlsim_coverage(ctx, _ptr(bitmap), 1 if clear else 0), ctx)


def rtlsim_get_mems(ctx, mems):
    _check(lib().rtlsim_get_mems(ctx, _ptr(mems)), ctx)


def rtlsim_reg_digest(ctx, digest):
    _check(lib().rtlsim_reg_digest(ctx, _ptr(digest)), ctx)


def rtlsim_stats(ctx) -> dict:
    st = Stats()
    _check(lib().rtlsim_stats(ctx, ctypes.byref(st)), ctx)
    return {f: getattr(st, f) for f, _ in Stats._fields_}


def rtlsim_launch_count(ctx) -> int:
    return int(lib().rtlsim_launch_count(ctx))


def rtlsim_last_error(ctx=None) -> str:
    m = lib().rtlsim_last_error(ctx)
    return m.decode() if m else ""


def rtlsim_free(ctx):
    lib().rtlsim_free(ctx)


# ------------------------------------------------------------ convenience --
class Simulator:
    """One loaded design on one device (one ctx)."""

    def __init__(self, ir, device=0, stream=None, op_lanes=0, chunk_cycles=0, flags=0, smem_limit=0):
        self.ir = ir
        self.flags = flags
        self.ctx = rtlsim_load(ir, device, stream, op_lanes, chunk_cycles, flags, smem_limit)
        st = self.stats()
        self.IW, self.OW, self.RW = st["iw"], st["ow"], st["rw"]
        self.N = self.T = 0
        self._keep = None

    def __del__(self, _free=rtlsim_free):
        if getattr(self, "ctx", None):
            try:
                _free(self.ctx)
            except Exception:   # interpreter shutdown: the process frees it
                pass
            self.ctx = None

    def stats(self) -> dict:
        return rtlsim_stats(self.ctx)

    def bind(self, stim: np.ndarray):
        stim = np.ascontiguousarray(stim, dtype=np.uint32)
        self._keep = stim
        rtlsim_bind(self.ctx, stim)
        self.N, self.T = stim.shape[0], stim.shape[1]

    def bind_device(self, stim_dev, N: int, T: int):
        self._keep = stim_dev
        rtlsim_bind_device(self.ctx, stim_dev, N, T)
        self.N, self.T = N, T

    def bind_stream(self, N: int, T: int, produce):
        """Producer binding: ``produce(c0, nc)`` returns the stimulus words
        [N][nc][IW] of cycles c0..c0+nc-1 (or None to abort the run)."""
        IW = self.IW

        def _cb(_user, c0, nc, dst):
            v = produce(int(c0), int(nc))
            if v is None:
                return 1
            n = N * int(nc) * IW
            if n:
                np.ctypeslib.as_array(dst, shape=(n,))[:] = np.asarray(v, np.uint32).reshape(-1)
            return 0

        cb = PRODUCER(_cb)
        self._keep = cb            # the library calls it during every run
        rtlsim_bind_stream(self.ctx, N, T, cb)
        self.N, self.T = N, T

    def run_stream(self, cycles: int, consume):
        """Consumer run: ``consume(c0, out[N][nc][OW], digest[N][nc] or None)``
        is called per chunk in cycle order; a false return aborts the run."""
        N, OW = self.N, self.OW

        def _cb(_user, c0, nc, out, dig):
            nc = int(nc)
            o = np.ctypeslib.as_array(out, shape=(N * nc * OW,)).reshape(N, nc, OW).copy() if N * nc * OW else \
                np.zeros((N, nc, OW), np.uint32)
            d = np.ctypeslib.as_array(dig, shape=(N * nc,)).reshape(N, nc).copy() if dig else None
            return 0 if consume(int(c0), o, d) else 1

        rtlsim_run_stream(self.ctx, cycles, CONSUMER(_cb))

    def run(self, cycles: int, out=True, regs=True, digest=False):
        o = np.zeros((self.N, cycles, self.OW), np.uint32) if out else None
        r = np.zeros((self.N, self.RW), np.uint32) if regs else None
        d = np.zeros((self.N, cycles), np.uint64) if digest else None
        rtlsim_run(self.ctx, cycles, o, r, d)
        return {"out": o, "regs": r, "digest": d}

    def run_device(self, cycles: int, out_dev=None, digest_dev=None):
        rtlsim_run_device(self.ctx, cycles, out_dev, digest_dev)

    def sync(self):
        rtlsim_sync(self.ctx)

    def get_regs(self) -> np.ndarray:
        r = np.zeros((self.N, self.RW), np.uint32)
        rtlsim_get_regs(self.ctx, r)
        return r

    def set_regs(self, regs: np.ndarray):
        rtlsim_set_regs(self.ctx, np.ascontiguousarray(regs, dtype=np.uint32))

    def reset(self):
        rtlsim_reset(self.ctx)

    def coverage(self, clear=False) -> np.ndarray:
        b = np.zeros(self.RW, np.uint32)
        rtlsim_coverage(self.ctx, b, clear)
        return b

    def get_mems(self) -> np.ndarray:
        m = np.zeros((self.N, int(getattr(self.ir, "MW", 0))), np.uint32)
        rtlsim_get_mems(self.ctx, m)
        return m

    def reg_digest(self) -> np.ndarray:
        d = np.zeros(self.N, np.uint64)
        rtlsim_reg_digest(self.ctx, d)
        return d

    def launch_count(self) -> int:
        return rtlsim_launch_count(self.ctx)
