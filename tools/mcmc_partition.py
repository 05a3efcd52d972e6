"""GPU-aware MCMC partitioning (Algorithm 1) on B200:
python tools/mcmc_partition.py <config> <n_tasks> <max_iter> [n_stim] [cycles]
(MCMC_SPLIT=1: split proposals — tasks are chunks of the op sequence, so
n_tasks above the IR's partition count splits partitions)
Prints one JSON line per iteration and a summary line: the cost (JIT evaluator
ms per cycle on n_stim stimuli) of the IR's own partitioning, of the all-ones
weights, and of the best graph the chain visited."""
import json
import os
import sys
import time

sys.path.insert(0, os.path.dirname(os.path.dirname(os.path.abspath(__file__))))
from rtlgen import shaped  # noqa: E402
from paper_conf_icpp_linrzkh22_b200 import partition as MP  # noqa: E402

cid = int(sys.argv[1])
n_tasks = int(sys.argv[2])
max_iter = int(sys.argv[3])
n_stim = int(sys.argv[4]) if len(sys.argv) > 4 else 4096
cycles = int(sys.argv[5]) if len(sys.argv) > 5 else 4
ir = shaped.generate(cid)
est = MP.gpu_estimator(n_stim=n_stim, cycles=cycles)
t0 = time.time()
c_orig = est(ir)
print(json.dumps({"cfg": cid, "what": "original partitions", "n_partitions": int(ir.n_partitions), "cost_ms": c_orig}), flush=True)
best, cost, hist = MP.mcmc_partition(ir, est, n_tasks=n_tasks, max_iter=max_iter, max_unimproved=max(5, max_iter // 3),
                                     beta=float(os.environ.get("MCMC_BETA", "20")), seed=1,
                                     split=os.environ.get("MCMC_SPLIT") == "1",
                                     log=lambda m: print(json.dumps({"log": m}), flush=True))
print(json.dumps({"cfg": cid, "split": os.environ.get("MCMC_SPLIT") == "1", "n_stim": n_stim, "cycles": cycles,
                  "n_tasks": n_tasks, "iterations": len(hist) - 1,
                  "cost_original_ms": c_orig, "cost_all_ones_ms": hist[0][1], "cost_best_ms": cost,
                  "best_n_partitions": int(best.n_partitions), "wall_s": round(time.time() - t0, 1),
                  "history": hist}), flush=True)
