"""Config-4 JIT parity on a small batch (env selects the variant)."""
import os, sys, json
import numpy as np
sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
import torch
import oracle
from rtlgen import shaped, stim
from paper_conf_icpp_linrzkh22_b200 import rtlsim as R
N = int(os.environ.get("BN", "2048")); C = int(os.environ.get("BC", "6"))
ir = shaped.generate(4)
seed = stim.STIM_SEED_BASE + 4
sim = R.Simulator(ir, chunk_cycles=C, flags=R.F_JIT)
d = stim.stimulus_torch(ir, seed, 0, N, 0, C)
out = torch.zeros((N, C, ir.OW), dtype=torch.int32, device="cuda")
sim.bind_device(d, N, C); sim.run_device(C, out); sim.sync()
regs = sim.get_regs()
pick = np.array([0, 1, 31, 32, 33, 100, 1000, N - 1])
st = stim.stimulus(ir, seed, pick, 0, C)
want = oracle.Design(ir).simulate(st, digest=False, threads=16)
go = out.cpu().numpy().view(np.uint32)[pick]
bad_out = np.argwhere(go != want["out"])
bad_reg = np.argwhere(regs[pick] != want["regs"])
print(json.dumps({"env": {k: v for k, v in os.environ.items() if k.startswith("RTLSIM_")}, "bad_out": len(bad_out),
                  "bad_reg": len(bad_reg), "first_out": bad_out[:4].tolist(), "first_reg": bad_reg[:6].tolist(),
                  "st": {k: sim.stats()[k] for k in ("smem_words", "n_steps", "op_lanes")}}), flush=True)
