"""Quick perf probe: eval-kernel time per cycle on the shaped configs."""
import os, sys, time, json
import numpy as np
import torch
sys.path.insert(0, '.')
from rtlgen import shaped, stim, designs
from paper_conf_icpp_linrzkh22_b200 import rtlsim as R

stream = torch.cuda.Stream()
torch.cuda.set_stream(stream)
cfgs = [int(x) for x in (sys.argv[1].split(',') if len(sys.argv) > 1 else ['2', '3', '4'])]
NS = {1: 1024, 2: 4096, 3: 16384, 4: 65536}
for cid in cfgs:
    t0 = time.time()
    ir = designs.tiny_dut() if cid == 1 else shaped.generate(cid)
    tg = time.time() - t0
    N = int(os.environ.get('N', NS[cid]))
    Tc = int(os.environ.get('TC', 4 if cid == 4 else 16))
    T = Tc * 4
    t0 = time.time()
    import os
    jit = (R.F_JIT if os.environ.get('JIT') else 0)
    sim = R.Simulator(ir, chunk_cycles=Tc, flags=R.F_TIMING | jit, op_lanes=int(os.environ.get('LANES', '0')), smem_limit=int(os.environ.get('SMEM_KB','0'))*1024, stream=torch.cuda.current_stream().cuda_stream)
    tl = time.time() - t0
    st = sim.stats()
    d_stim = stim.stimulus_torch(ir, stim.STIM_SEED_BASE + cid, 0, N, 0, T)
    out = torch.empty((N, Tc, ir.OW), dtype=torch.int32, device='cuda')
    sim.bind_device(d_stim, N, T)
    sim.run_device(Tc, out)   # warm
    sim.sync()
    s0 = sim.stats()
    e0, e1 = torch.cuda.Event(True), torch.cuda.Event(True)
    e0.record()
    for _ in range(3):
        sim.run_device(Tc, out)
    e1.record(); torch.cuda.synchronize()
    ms = e0.elapsed_time(e1)
    s1 = sim.stats()
    ems = s1['eval_ms'] - s0['eval_ms']
    stc = 3 * Tc * N
    print(json.dumps({"cfg": cid, "env": {k: os.environ.get(k) for k in ("JIT","LANES","SMEM_KB","RTLSIM_JIT_OPT","RTLSIM_JIT_TMAX","RTLSIM_JIT_TPC","N")}, "tpc_max_smem": 232448 // max(1, st["smem_words"]*4), "jit_s": s1["jit_compile_s"], "cubin": s1["jit_cubin_bytes"], "tpc_used": None, "gen_s": round(tg,1), "load_s": round(tl,2), "L": st['op_lanes'], "smem_KB": st['smem_words']*4/1024,
          "steps": st['n_steps'], "desc": st['n_desc'], "b_floor": st['b_floor'], "b_state": st['b_state'],
          "ms_per_cycle_total": ms / (3*Tc), "ms_per_cycle_eval": ems / (3*Tc),
          "stim_cyc_per_s": stc / (ms/1e3), "sass": s1["jit_sass_instructions"], "tmem_cols": s1["tmem_cols"],
          "warp_instr_per_s": s1["jit_sass_instructions"] * (N / 32) / (ems / (3*Tc) / 1e3) if s1["jit_sass_instructions"] else None, "eval_GBps_floor": st['b_floor'] * stc / (ems/1e3) / 1e9}))
