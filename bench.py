#!/usr/bin/env python
"""bench.py — stimulus-cycles/s of the B200 batch-stimulus RTL simulator.

Workload (BASELINE.json configs[3], the north star's headline): the
NVDLA-shaped synthetic design (1,048,576 ops, 64 partitions, seeded), 65536
stimuli per GPU. A "step" is one pass of the whole hot path over one batch:
`--cycles-per-step` clock cycles of every stimulus (stimulus transpose N2,
evaluation of every partition's ops N1, register update, output transpose N3).
Stimulus and outputs stay in HBM for `value`; `e2e` repeats the measurement
through the C ABI with pinned HOST buffers (H2D + D2H inside the timed region).

Multi-GPU (one process per GPU under torchrun, NCCL): config 5 — the 262144
stimuli of BASELINE.json configs[4] in contiguous blocks of 262144/G per GPU
(strong scaling; --stimuli-per-gpu K switches to weak scaling). The run goes
through paper_conf_icpp_linrzkh22_b200.parallel.run_sharded, the harness the
gloo tests cover: no collective inside the timed region, the elapsed time is
the max over ranks, and the per-stimulus register digests (N x 8 B) are
gathered to rank 0 after timing.

`--impl reference` times the CPU oracle (oracle/liboracle.so), the only
reference this tier has, on a bounded sample of the same workload.
"""
from __future__ import annotations

import argparse
import json
import os
import statistics
import sys
import threading
import time

import numpy as np

ROOT = os.path.dirname(os.path.abspath(__file__))
sys.path.insert(0, ROOT)

from rtlgen import designs, shaped, stim  # noqa: E402

CONFIG_NAMES = {1: "tiny", 2: "riscv-mini-shaped", 3: "spinal-shaped", 4: "nvdla-shaped"}
CONFIG_N = {1: 1024, 2: 4096, 3: 16384, 4: 65536}
CONFIG5_N = 262144   # config 5: the NVDLA-shaped design sharded over 2/4/8 GPUs


def parse():
    ap = argparse.ArgumentParser()
    ap.add_argument("--gpus", type=int, default=1)
    ap.add_argument("--steps", type=int, default=10)
    ap.add_argument("--warmup", type=int, default=3)
    ap.add_argument("--impl", default="ours", choices=["ours", "reference"])
    ap.add_argument("--config", type=int, default=4, choices=[1, 2, 3, 4])
    ap.add_argument("--stimuli-per-gpu", type=int, default=0)
    ap.add_argument("--cycles-per-step", type=int, default=0)
    ap.add_argument("--no-e2e", action="store_true")
    ap.add_argument("--no-cpu-baseline", action="store_true")
    ap.add_argument("--graph", action="store_true", help="per-(cycle, partition) CUDA-graph schedule")
    ap.add_argument("--backend", default="jit", choices=["jit", "interp"],
                    help="jit: specialized per-partition kernels (RTLSIM_F_JIT); interp: the op-stream interpreter")
    return ap.parse_args()


def make_design(cid):
    return designs.tiny_dut() if cid == 1 else shaped.generate(cid)


def peaks():
    p = os.path.join(ROOT, "MEASURED_PEAKS.json")
    if os.path.exists(p):
        d = json.load(open(p))
        return float(d["hbm_gbs"]), "measured (MEASURED_PEAKS.json hbm_gbs, copy)"
    return 6650.0, "fallback (B200_PROFILING.md: 6.65 TB/s)"


class ClockSampler:
    """NVML SM clock + throttle reasons during the timed region."""

    def __init__(self, dev_index):
        self.samples, self.reasons, self.max_mhz = [], set(), None
        self._stop = threading.Event()
        try:
            import pynvml
            pynvml.nvmlInit()
            self.nv = pynvml
            self.h = pynvml.nvmlDeviceGetHandleByIndex(dev_index)
            self.max_mhz = pynvml.nvmlDeviceGetMaxClockInfo(self.h, pynvml.NVML_CLOCK_SM)
        except Exception:
            self.nv = None
        self._t = threading.Thread(target=self._run, daemon=True)

    def _run(self):
        nv = self.nv
        names = {"hw_slowdown": 0x8, "sw_thermal_slowdown": 0x20, "hw_thermal_slowdown": 0x40,
                 "sw_power_cap": 0x4, "hw_power_brake_slowdown": 0x80}
        while not self._stop.is_set():
            try:
                self.samples.append(nv.nvmlDeviceGetClockInfo(self.h, nv.NVML_CLOCK_SM))
                r = nv.nvmlDeviceGetCurrentClocksEventReasons(self.h)
                for k, bit in names.items():
                    if r & bit:
                        self.reasons.add(k)
            except Exception:
                pass
            time.sleep(0.1)

    def __enter__(self):
        if self.nv:
            self._t.start()
        return self

    def __exit__(self, *a):
        self._stop.set()
        if self.nv and self._t.is_alive():
            self._t.join()

    def summary(self):
        return {"sm_mhz": statistics.median(self.samples) if self.samples else None,
                "sm_max_mhz": self.max_mhz, "reasons": sorted(self.reasons), "samples": len(self.samples)}


def cpu_oracle_rate(ir, cid, seed, budget_s=15.0, single_s=10.0):
    """The oracle as it stands on a bounded sample of the same workload
    (stimuli 0..S-1, cycles 0..C-1): multi-threaded over stimuli on all host
    cores for ~budget_s, and single-threaded for >= single_s seconds."""
    import oracle
    d = oracle.Design(ir)
    cores = len(os.sched_getaffinity(0))

    def sample(S, C):
        if cid == 1:
            return stim.tiny_stimulus(seed, np.arange(S), 100, 0, C)
        return stim.stimulus(ir, seed, np.arange(S), 0, C)
    # calibrate on one stimulus-cycle
    t = time.perf_counter()
    d.simulate(sample(1, 1), out=False, regs=False, threads=1)
    per = max(time.perf_counter() - t, 1e-6)
    # single thread, >= single_s seconds of simulation
    n1 = max(1, int(single_s / per))
    C1 = max(1, min(100, int(np.sqrt(n1))))
    S1 = max(1, -(-n1 // C1))
    st1 = sample(S1, C1)
    t = time.perf_counter()
    d.simulate(st1, out=True, regs=True, threads=1)
    el1 = time.perf_counter() - t
    # all cores
    total = max(cores, int(budget_s * cores / per))
    C = max(1, min(100, int(np.sqrt(total / cores))))
    S = max(cores, total // C)
    st = sample(S, C)
    t = time.perf_counter()
    d.simulate(st, out=True, regs=True, threads=cores)
    el = time.perf_counter() - t
    return {"value": S * C / el, "unit": "stimulus-cycles/s", "cores": cores, "kind": "oracle",
            "sample": f"{S} stimuli x {C} cycles of the same design/seed, multi-threaded over stimuli "
                      f"({el:.1f} s)",
            "single_thread_value": S1 * C1 / el1,
            "single_thread_sample": f"{S1} stimuli x {C1} cycles, 1 thread ({el1:.1f} s)",
            "host": host_info()}


def run_reference(a):
    rank = int(os.environ.get("RANK", "0"))
    if rank != 0:
        return
    cid = a.config
    ir = make_design(cid)
    seed = stim.STIM_SEED_BASE + cid
    import oracle
    d = oracle.Design(ir)
    cores = len(os.sched_getaffinity(0))
    st1 = stim.stimulus(ir, seed, [0], 0, 1)
    t = time.perf_counter()
    d.simulate(st1, out=False, regs=False, threads=1)
    per = max(time.perf_counter() - t, 1e-6)
    # each step: a sample sized so that W + K steps take ~2 minutes in total
    per_step = 120.0 / max(1, a.steps + a.warmup)
    S = max(cores, int(per_step * cores / per))
    st = stim.stimulus(ir, seed, np.arange(S), 0, 1)
    for _ in range(a.warmup):
        d.simulate(st, threads=cores)
    t = time.perf_counter()
    for _ in range(a.steps):
        d.simulate(st, threads=cores)
    el = time.perf_counter() - t
    v = S * a.steps / el
    line = {"metric": "stimulus-cycles/sec", "value": v, "unit": "stimulus-cycles/s", "impl": "reference",
            "n_gpus": a.gpus, "steps": a.steps, "warmup": a.warmup, "ms_per_step": el / a.steps * 1e3,
            "higher_is_better": True, "scaling": "weak", "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {"workload": f"{CONFIG_NAMES[cid]} (config {cid}): CPU oracle on a bounded sample",
                       "stimuli_per_step": S, "cycles_per_step": 1},
            "cpu_baseline": {"value": v, "unit": "stimulus-cycles/s", "cores": cores, "kind": "oracle",
                             "sample": f"{S} stimuli x 1 cycle per step", "host": host_info()},
            "e2e": {"value": v, "unit": "stimulus-cycles/s", "h2d_bytes_per_step": 0, "d2h_bytes_per_step": 0}}
    print(json.dumps(line), flush=True)


def host_info():
    """CPU model, logical cores available to this process and RAM (for the
    cpu_baseline record)."""
    model = None
    try:
        for line in open("/proc/cpuinfo"):
            if line.startswith("model name"):
                model = line.split(":", 1)[1].strip()
                break
    except OSError:
        pass
    ram = None
    try:
        for line in open("/proc/meminfo"):
            if line.startswith("MemTotal"):
                ram = round(int(line.split()[1]) / 1024 / 1024, 1)
                break
    except OSError:
        pass
    return {"cpu_model": model, "cores": len(os.sched_getaffinity(0)), "ram_gb": ram}


def run_ours(a):
    import torch
    import torch.distributed as dist
    from paper_conf_icpp_linrzkh22_b200 import build, parallel, rtlsim as R

    world = int(os.environ.get("WORLD_SIZE", "1"))
    rank = int(os.environ.get("RANK", "0"))
    # RTLSIM_BENCH_BACKEND=gloo (tests only): several ranks on one GPU, CPU
    # collectives — exercises the multi-rank path where only one GPU exists
    backend = os.environ.get("RTLSIM_BENCH_BACKEND", "nccl")
    local = int(os.environ.get("LOCAL_RANK", "0")) % max(1, torch.cuda.device_count())
    if world > 1:
        if backend == "nccl":
            dist.init_process_group("nccl", device_id=torch.device("cuda", local))
        else:
            dist.init_process_group(backend)
    coll_dev = "cuda" if backend == "nccl" else "cpu"
    torch.cuda.set_device(local)

    def staged(fn):
        # the node's local rank 0 first (nvcc build, JIT compile into the
        # shared cubin cache), then the other ranks (cache hits)
        if world > 1 and local != 0:
            dist.barrier()
        r = fn()
        if world > 1 and local == 0:
            dist.barrier()
        return r

    os.environ.setdefault("RTLSIM_JIT_CACHE", f"/tmp/rtlsim_jit_cache-{os.getuid()}")
    staged(build.build)
    cid = a.config
    # N=1: config 4 (65536 stimuli). N>1: config 5 — 262144 stimuli in total
    # over the G GPUs (strong scaling, 262144/G per GPU), unless
    # --stimuli-per-gpu asks for weak scaling.
    if a.stimuli_per_gpu:
        n_total, scaling = a.stimuli_per_gpu * world, "weak"
    elif world > 1 and cid == 4:
        n_total, scaling = CONFIG5_N, "strong"
    else:
        n_total, scaling = CONFIG_N[cid] * world, "weak"
    Tc = a.cycles_per_step or (10 if cid == 4 else 100)
    ir = make_design(cid)
    seed = stim.STIM_SEED_BASE + cid
    stream = torch.cuda.Stream()
    torch.cuda.set_stream(stream)
    flags = R.F_TIMING | (R.F_GRAPH if a.graph else 0) | (R.F_JIT if a.backend == "jit" else 0)
    info = {}

    def simulate(s0, N):
        """This rank's shard [s0, s0+N): device-resident stimulus, W warm-up
        steps, K timed steps between CUDA events on the launching stream, then
        (after timing) the per-stimulus register digests for the rank-0 gather
        and the pinned-host e2e measurement."""
        t_load = time.perf_counter()
        sim = staged(lambda: R.Simulator(ir, device=local, stream=stream.cuda_stream, chunk_cycles=Tc,
                                         flags=flags))
        info["load_s"] = time.perf_counter() - t_load
        T = (a.warmup + a.steps) * Tc
        if cid == 1:
            host = stim.tiny_stimulus(seed, np.arange(s0, s0 + N), T)
            d_stim = torch.from_numpy(host.view(np.int32)).cuda()
        else:
            d_stim = torch.empty((N, T, ir.IW), dtype=torch.int32, device="cuda")
            for c0 in range(0, T, Tc):     # generate in chunks to bound temporaries
                d_stim[:, c0:c0 + Tc] = stim.stimulus_torch(ir, seed, s0, N, c0, min(Tc, T - c0))
        out = torch.empty((N, Tc, ir.OW), dtype=torch.int32, device="cuda")
        sim.bind_device(d_stim, N, T)

        def first_run():   # JIT kernels are compiled here, specialised for N_pad
            sim.run_device(Tc, out)
            sim.sync()
        t_jit = time.perf_counter()
        staged(first_run)
        info["first_run_s"] = time.perf_counter() - t_jit
        for _ in range(a.warmup - 1):
            sim.run_device(Tc, out)
        sim.sync()
        torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        s_before = sim.stats()
        l_before = sim.launch_count()
        e0, e1 = torch.cuda.Event(enable_timing=True), torch.cuda.Event(enable_timing=True)
        with ClockSampler(local) as clk:
            e0.record(stream)
            for _ in range(a.steps):
                sim.run_device(Tc, out)
            e1.record(stream)
            torch.cuda.synchronize()
        if world > 1:
            dist.barrier()
        ms = e0.elapsed_time(e1)
        info.update(stats=sim.stats(), s_before=s_before, launches=sim.launch_count() - l_before,
                    clocks=clk.summary(), ms=ms, N=N)
        # after timing: the final register state of every stimulus, as digests
        reg_dig = sim.reg_digest()
        # e2e: the same metric through the C ABI with pinned HOST buffers
        if not a.no_e2e:
            h_stim = d_stim.cpu().pin_memory()
            del d_stim
            h_out = torch.empty((N, Tc, ir.OW), dtype=torch.int32).pin_memory()
            R.rtlsim_bind(sim.ctx, h_stim.numpy())
            for _ in range(a.warmup):
                R.rtlsim_run(sim.ctx, Tc, h_out.numpy(), None, None)
            if world > 1:
                dist.barrier()
            t = time.perf_counter()
            for _ in range(a.steps):
                R.rtlsim_run(sim.ctx, Tc, h_out.numpy(), None, None)
            el = torch.tensor([time.perf_counter() - t], dtype=torch.float64, device=coll_dev)
            if world > 1:
                dist.all_reduce(el, op=dist.ReduceOp.MAX)
            info["e2e_s"] = float(el.item())
        del sim
        return {"elapsed": ms / 1e3, "reg_digest": reg_dig, "coverage": None}

    res = parallel.run_sharded(simulate, n_total, device=coll_dev)
    st, s_before, ms, N = info["stats"], info["s_before"], info["ms"], info["N"]
    ms_max = res.elapsed_max * 1e3
    total = n_total * Tc * a.steps
    value = total / (ms_max / 1e3)

    # roofline of the dominant kernel (the evaluator), measured live
    ev_ms = st["eval_ms"] - s_before["eval_ms"]
    ev_n = st["eval_launches"] - s_before["eval_launches"]
    ev_sc = st["eval_stim_cycles"] - s_before["eval_stim_cycles"]
    avg_ms = ev_ms / max(ev_n, 1)
    bytes_per_launch = st["b_floor"] * ev_sc / max(ev_n, 1)
    achieved = bytes_per_launch / (avg_ms / 1e3) / 1e9
    peak, peak_src = peaks()
    traffic = None
    prof = os.path.join(ROOT, "profiles", f"ncu_config{cid}.json")
    if os.path.exists(prof):
        pj = json.load(open(prof))
        if pj.get("dram_bytes_per_stim_cycle"):
            traffic = pj["dram_bytes_per_stim_cycle"] * ev_sc / max(ev_n, 1)
    e2e = None
    if "e2e_s" in info:
        e2e = {"value": total / info["e2e_s"], "unit": "stimulus-cycles/s",
               "h2d_bytes_per_step": N * Tc * ir.IW * 4, "d2h_bytes_per_step": N * Tc * ir.OW * 4,
               "path": "rtlsim_bind(pinned host stim) + rtlsim_run(cycles, pinned host out)"}

    cpu = None
    if rank == 0 and world == 1 and not a.no_cpu_baseline:
        cpu = cpu_oracle_rate(ir, cid, seed)

    if rank == 0:
        dig = res.reg_digest
        line = {
            "metric": "stimulus-cycles/sec", "value": value, "unit": "stimulus-cycles/s",
            "n_gpus": world, "steps": a.steps, "warmup": a.warmup, "ms_per_step": ms_max / a.steps,
            "higher_is_better": True, "scaling": scaling, "vs_baseline": None, "dtype": "u32",
            "data": "synthetic",
            "config": {
                "workload": (f"{CONFIG_NAMES[cid]} (config {5 if scaling == 'strong' else cid}): "
                             f"{st['n_ops']} ops ({st['n_live_ops']} live after dead-logic elimination), "
                             f"{st['n_partitions']} partitions, {n_total} stimuli over {world} GPU(s) "
                             f"x {Tc} cycles per step"),
                "stimuli_total": n_total, "stimuli_per_gpu": N, "cycles_per_step": Tc,
                "n_ops": st["n_ops"], "n_live_ops": st["n_live_ops"], "word_ops": st["word_ops"],
                "live_word_ops": st["live_word_ops"],
                "op_lanes": st["op_lanes"], "tiles_per_cta": st["jit_tiles_per_cta"],
                "warps_per_cta": st["op_lanes"] * max(1, st["jit_tiles_per_cta"]),
                "sass_instructions": st["jit_sass_instructions"],
                "warp_instructions_per_live_op": (st["jit_sass_instructions"] / max(1, st["n_live_ops"])
                                                  if st["jit_sass_instructions"] else None),
                "warps_sharing_each_fetched_instruction": st["jit_tiles_per_cta"] or None,
                "tmem_cols_per_tile": st["tmem_cols"],
                "value_tiers": ("shared memory + TMEM (computed U32 values, tcgen05.ld/st)" if st["tmem_cols"]
                                else "shared memory"),
                "design_seed": hex(stim.DESIGN_SEED_BASE + cid), "stim_seed": hex(seed),
                "parallelism": f"contiguous stimulus shards x{world} (parallel.run_sharded)",
                "schedule": "jit per-(cycle, partition) kernels, graph-launched" if a.backend == "jit"
                            else ("graph" if a.graph else "fused interpreter"),
                "backend": a.backend, "load_s": round(info["load_s"], 1),
                "jit_compile_s": round(st["jit_compile_s"], 1), "first_run_s": round(info["first_run_s"], 1),
                "l2": f"register state {st['b_floor'] * N / 2 / 1e9:.1f} GB per buffer >> 126 MB L2 (no flush needed)",
                "final_reg_digest_xor": None if dig is None else hex(int(np.bitwise_xor.reduce(dig))),
                "final_reg_digests_gathered": None if dig is None else int(dig.size),
            },
            "roofline": {"bound": "hbm", "achieved": achieved, "peak": peak, "unit": "GB/s",
                         "frac": achieved / peak, "traffic": traffic,
                         "kernel": "rtl_jit_part (one per partition per cycle)" if a.backend == "jit"
                                   else "rtl_eval_kernel",
                         "peak_source": peak_src,
                         "algorithmic_bytes_per_stim_cycle": st["b_floor"],
                         # the timed unit is one graph launch: cycles_per_step x partitions kernel nodes
                         "eval_ms_per_graph_launch": avg_ms,
                         "kernel_nodes_per_graph_launch": Tc * st["n_partitions"] if a.backend == "jit" else None,
                         "eval_share_of_step": ev_ms / max(ms, 1e-9),
                         "traffic_source": "profiles/ncu_config%d.json (ncu DRAM bytes of one full cycle)" % cid},
            "cpu_baseline": cpu, "e2e": e2e, "gpu_launches": info["launches"], "clocks": info["clocks"],
        }
        print(json.dumps(line), flush=True)
    if world > 1:
        dist.destroy_process_group()


def main():
    a = parse()
    if a.impl == "reference":
        run_reference(a)
    else:
        run_ours(a)


if __name__ == "__main__":
    main()
