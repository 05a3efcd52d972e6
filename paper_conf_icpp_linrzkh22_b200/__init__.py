"""B200-native batch-stimulus RTL simulation (the hot path of RTLflow, ICPP'22).

The product is librtlsim.so (C ABI: include/rtlsim.h) built from csrc/ for
sm_100a; :mod:`.rtlsim` is its thin ctypes binding and :mod:`.parallel`
the torch.distributed stimulus-sharding harness.
"""
from .rtlsim import Simulator, RtlsimError  # noqa: F401
