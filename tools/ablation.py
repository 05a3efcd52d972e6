"""Runtime ablations of SURVEY §8(f) row 2 (Table 4 and Table 5) on B200.

Table 4: the same per-(cycle, partition) schedule issued as
individual stream launches (RTLSIM_F_STREAM) vs captured once in a CUDA graph
(RTLSIM_F_GRAPH) — plus this build's fused chunk kernel (default) and the JIT
backend (RTLSIM_F_JIT, graph-launched).
Table 5: host-buffer runs (stimulus upload + output drain in
the timed region) with the chunk pipeline vs serialised (RTLSIM_F_NO_PIPELINE).

python tools/ablation.py <config> [N] [cycles]   -> one JSON line per variant
"""
import json
import os
import sys
import time

import numpy as np
import torch

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from rtlgen import designs, shaped, stim  # noqa: E402
from paper_conf_icpp_linrzkh22_b200 import rtlsim as R  # noqa: E402

cid = int(sys.argv[1]) if len(sys.argv) > 1 else 3
NDEF = {1: 1024, 2: 4096, 3: 16384, 4: 65536}
N = int(sys.argv[2]) if len(sys.argv) > 2 else NDEF[cid]
T = int(sys.argv[3]) if len(sys.argv) > 3 else 64
Tc = 16
ir = designs.tiny_dut() if cid == 1 else shaped.generate(cid)
seed = stim.STIM_SEED_BASE + cid
d_stim = stim.stimulus_torch(ir, seed, 0, N, 0, T) if cid != 1 else torch.from_numpy(
    stim.tiny_stimulus(seed, np.arange(N), T).view(np.int32)).cuda()


def device_run(flags, reps=2):
    sim = R.Simulator(ir, chunk_cycles=Tc, flags=flags)
    out = torch.empty((N, Tc, ir.OW), dtype=torch.int32, device="cuda")
    sim.bind_device(d_stim, N, T)
    sim.run_device(Tc, out)   # warm-up (graph capture, JIT load)
    sim.sync()
    best = None
    for _ in range(reps):
        R.rtlsim_reset(sim.ctx)
        torch.cuda.synchronize()
        t = time.perf_counter()
        for _ in range(T // Tc):
            sim.run_device(Tc, out)
        sim.sync()
        el = time.perf_counter() - t
        best = el if best is None else min(best, el)
    return N * T / best


def host_run(flags, reps=2):
    sim = R.Simulator(ir, chunk_cycles=Tc, flags=flags)
    h_stim = d_stim.cpu().numpy().view(np.uint32)
    h_out = np.empty((N, T, ir.OW), np.uint32)
    R.rtlsim_bind(sim.ctx, h_stim)
    R.rtlsim_run(sim.ctx, Tc, h_out[:, :Tc], None, None)   # warm-up
    best = None
    for _ in range(reps):
        R.rtlsim_reset(sim.ctx)
        t = time.perf_counter()
        R.rtlsim_run(sim.ctx, T, h_out, None, None)
        el = time.perf_counter() - t
        best = el if best is None else min(best, el)
    return N * T / best


variants = [
    ("fused interpreter (default)", "device", 0),
    ("graph: per-(cycle,partition) interpreter nodes", "device", R.F_GRAPH),
    ("stream: per-(cycle,partition) interpreter launches", "device", R.F_STREAM),
    ("jit (graph-launched)", "device", R.F_JIT),
    ("jit stream-launched", "device", R.F_JIT | R.F_STREAM),
    ("host buffers, jit, pipelined (default)", "host", R.F_JIT),
    ("host buffers, jit, no pipeline", "host", R.F_JIT | R.F_NO_PIPELINE),
]
if len(sys.argv) > 4:
    variants = [v for v in variants if sys.argv[4] in v[0]]
for name, kind, flags in variants:
    try:
        v = device_run(flags) if kind == "device" else host_run(flags)
        print(json.dumps({"config": cid, "N": N, "cycles": T, "variant": name, "stim_cycles_per_s": v}), flush=True)
    except Exception as e:   # report and continue
        print(json.dumps({"config": cid, "variant": name, "error": str(e)[:200]}), flush=True)
