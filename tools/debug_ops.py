"""Debug helper: single-op designs per opcode x widths on the GPU vs the oracle."""
import sys, itertools
import numpy as np
sys.path.insert(0, '.')
import oracle
from rtlgen import ir as I, stim, designs
from rtlgen.builder import Builder
from paper_conf_icpp_linrzkh22_b200 import rtlsim as R

def one(name, wd, wa, wb=0, wc=0, imm=0, const_b=None):
    b = Builder(name)
    a = b.input(wa)
    bb = b.input(wb) if wb and const_b is None else (b.const(wb, const_b) if wb else None)
    cc = b.input(wc) if wc else None
    d = b.op(name, wd, a, bb, cc, imm=imm)
    b.output(d)
    return b.build()

bad = 0
for name in I.OPCODES:
    for wd, wa in [(1,1),(4,4),(1,5),(8,3),(16,16),(12,20),(32,32),(33,40),(64,64),(100,70),(5,100)]:
        if name in I.MULDIV and max(wd, wa) > 64: continue
        wb = 3 if name in I.SHIFTS else (wa if name not in I.UNARY else 0)
        wc = wa if name == "MUX" else 0
        imm = 0
        if name == "SLICE":
            if wd > wa: continue
            imm = wa - wd
        for cb in (None, 5) if wb else (None,):
            ir = one(name, wd, wa, wb, wc, imm, cb)
            st = stim.stimulus(ir, 7, np.arange(64), 0, 3)
            want = oracle.simulate(ir, st)["out"]
            sim = R.Simulator(ir)
            sim.bind(st)
            got = sim.run(3)["out"]
            if not np.array_equal(got, want):
                bad += 1
                i = np.argwhere(got != want)[0]
                print("MISMATCH", name, wd, wa, wb, wc, "const" if cb else "", "at", i.tolist(), got[tuple(i)], want[tuple(i)], st[i[0], i[1]])
print("bad", bad)
