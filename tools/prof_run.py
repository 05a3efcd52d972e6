"""One short evaluator launch for ncu: python tools/prof_run.py <config> <cycles_per_launch> <launches>"""
import sys
import torch
sys.path.insert(0, '.')
from rtlgen import shaped, stim, designs
from paper_conf_icpp_linrzkh22_b200 import rtlsim as R

cid = int(sys.argv[1]); Tc = int(sys.argv[2]); nl = int(sys.argv[3]) if len(sys.argv) > 3 else 2
NS = {1: 1024, 2: 4096, 3: 16384, 4: 65536}
ir = designs.tiny_dut() if cid == 1 else shaped.generate(cid)
import os
N = int(os.environ.get('PROF_N', NS[cid]))
s = torch.cuda.Stream(); torch.cuda.set_stream(s)
flags = (R.F_JIT if os.environ.get('JIT') else 0)
sim = R.Simulator(ir, chunk_cycles=Tc, stream=s.cuda_stream, flags=flags, op_lanes=int(os.environ.get('LANES', '0')), smem_limit=int(os.environ.get('SMEM_KB','0'))*1024)
d_stim = stim.stimulus_torch(ir, stim.STIM_SEED_BASE + cid, 0, N, 0, Tc * nl)
out = torch.empty((N, Tc, ir.OW), dtype=torch.int32, device='cuda')
sim.bind_device(d_stim, N, Tc * nl)
for _ in range(nl):
    sim.run_device(Tc, out)
sim.sync()
print("done", sim.stats()["smem_words"])
