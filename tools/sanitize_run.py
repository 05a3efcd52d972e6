"""Small runs for compute-sanitizer (memcheck / racecheck / synccheck): the tiny
DUT and a reduced riscv-mini-shaped design on the JIT and interpreter paths,
checked against the oracle. Exit code 0 iff every result matches."""
import os
import sys

import numpy as np

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import oracle  # noqa: E402
from rtlgen import designs, shaped, stim  # noqa: E402
from paper_conf_icpp_linrzkh22_b200 import rtlsim as R  # noqa: E402

ok = True
cases = [(designs.tiny_dut(), stim.tiny_stimulus(stim.STIM_SEED_BASE + 1, np.arange(64), 8, mode="B"))]
ir2 = shaped.generate(2, scale=0.05)
cases.append((ir2, stim.stimulus(ir2, stim.STIM_SEED_BASE + 2, np.arange(64), 0, 4)))
for ir, st in cases:
    want = oracle.simulate(ir, st, digest=True)
    for fl in (R.F_JIT, 0):
        sim = R.Simulator(ir, chunk_cycles=4, flags=fl)
        sim.bind(st)
        got = sim.run(st.shape[1], out=True, regs=True, digest=True)
        for k in ("out", "regs", "digest"):
            if not np.array_equal(got[k], want[k]):
                print("MISMATCH", ir.name, fl, k)
                ok = False
        del sim
print("sanitize_run", "ok" if ok else "FAILED")
sys.exit(0 if ok else 1)
