"""GPU-aware partitioning by MCMC — PAPER.md §3.2.1, Algorithm 1,
Eq 1-3; SURVEY §8(f) row 1.

The paper feeds a weight vector over the k most frequent RTL node types into
Verilator's merge-based partitioner (Eq 1: weight_sum(task) = sum_t w_t N_t)
and searches the weights with Metropolis-Hastings (Eq 2: p(G) ~ exp(-beta
cost(G)); Eq 3: a(G -> G*) = min(1, exp(beta (cost(G) - cost(G*))))), the
cost of a proposed task graph G being measured by compiling and running it on
the GPU with a few stimuli and cycles (the estimator).

Here the tasks being merged are the partitions the IR arrives with (the
levelized design's macro tasks): `propose` walks them in a
topological order of the partition DAG and merges consecutive ones into a task
while the task's weight_sum stays under total / n_tasks — weights change where
the task boundaries fall, and so the B200 schedule (steps per cycle, shared-
memory working set, cross-partition nets, launches per cycle). The estimator
is the production path (`rtlsim_load` with the JIT backend + `rtlsim_run` on
`n_stim` device-resident stimuli for `cycles` cycles, CUDA-event timed);
tests substitute any callable. Results never depend on the partitioning
(reading 16): only the schedule changes.

Host-side orchestration only: every simulation runs through the C ABI.
"""
from __future__ import annotations

import dataclasses
import math
import random
from typing import Callable

import numpy as np

UNUSED = 0xFFFFFFFF


def _wclass(w: np.ndarray) -> np.ndarray:
    return np.where(w == 1, 0, np.where(w <= 8, 1, np.where(w <= 16, 2, np.where(w <= 32, 3, 4))))


def node_types(ir) -> np.ndarray:
    """Per-op RTL node type: (opcode, destination width class)."""
    return ir.ops["opcode"].astype(np.int64) * 5 + _wclass(ir.width[ir.ops["dst"]].astype(np.int64))


def top_types(ir, k: int = 30) -> np.ndarray:
    """T of Eq 1: the k most frequent node types (ties by type id)."""
    t, n = np.unique(node_types(ir), return_counts=True)
    order = np.lexsort((t, -n))
    return t[order[:k]]


def partition_order(ir) -> list[int]:
    """A topological order of the IR's partition DAG (ties by partition id)."""
    P = int(ir.n_partitions)
    drv = np.full(len(ir.width), -1, np.int64)
    drv[ir.ops["dst"]] = ir.ops["part"]
    succ = [set() for _ in range(P)]
    for f in ("a", "b", "c"):
        src = ir.ops[f]
        ok = src != UNUSED
        sp = drv[src[ok]]
        dp = ir.ops["part"][ok].astype(np.int64)
        m = (sp >= 0) & (sp != dp)
        for p, q in set(zip(sp[m].tolist(), dp[m].tolist())):
            succ[p].add(q)
    indeg = [0] * P
    for p in range(P):
        for q in succ[p]:
            indeg[q] += 1
    import heapq
    h = [p for p in range(P) if indeg[p] == 0]
    heapq.heapify(h)
    out = []
    while h:
        p = heapq.heappop(h)
        out.append(p)
        for q in sorted(succ[p]):
            indeg[q] -= 1
            if indeg[q] == 0:
                heapq.heappush(h, q)
    if len(out) != P:
        raise ValueError("partition DAG has a cycle")
    return out


@dataclasses.dataclass
class Optimizer:
    """Algorithm 1's optimizer: weights over T, proposal = a task graph.

    split=False: tasks merge consecutive IR partitions (topological order).
    split=True: tasks are contiguous chunks of the global op sequence (IR
    partitions in topological order, each partition's ops in topological
    order), cut where the running weight_sum crosses multiples of
    total / n_tasks — a cut may fall inside an IR partition, so n_tasks above
    the IR's partition count splits partitions: smaller per-task working sets
    (more tiles per CTA on the B200) for more cross-task nets (HBM bytes).
    Contiguous chunks of a topological order keep the task graph acyclic."""
    ir: object
    n_tasks: int
    k: int = 30
    step: float = 1.0
    seed: int = 0
    split: bool = False

    def __post_init__(self):
        self.T = top_types(self.ir, self.k)
        self.types = node_types(self.ir)
        self.order = partition_order(self.ir)
        self.rng = random.Random(self.seed)
        P = int(self.ir.n_partitions)
        # N_t per (partition, type in T); types outside T weigh 1 (fixed)
        self.count = np.zeros((P, len(self.T)), np.int64)
        self.other = np.zeros(P, np.int64)
        idx = {int(t): j for j, t in enumerate(self.T)}
        col = np.array([idx.get(int(t), -1) for t in self.types])
        parts = self.ir.ops["part"].astype(np.int64)
        ok = col >= 0
        np.add.at(self.count, (parts[ok], col[ok]), 1)
        np.add.at(self.other, parts[~ok], 1)
        self.initialize_weights()

    # line 5
    def initialize_weights(self):
        self.weights = np.ones(len(self.T))
        self.candidate = self.weights.copy()

    # line 7: randomly increase one weight of the current vector
    def random_increase(self):
        self.candidate = self.weights.copy()
        self.candidate[self.rng.randrange(len(self.T))] += self.step

    # Eq 1 per IR partition
    def weight_sum(self, w: np.ndarray) -> np.ndarray:
        return self.count @ w + self.other

    # Eq 1 per op (weights of the op's node type; 1 outside T)
    def op_weights(self, w: np.ndarray) -> np.ndarray:
        idx = {int(t): j for j, t in enumerate(self.T)}
        col = np.array([idx.get(int(t), -1) for t in self.types])
        return np.where(col >= 0, w[np.maximum(col, 0)], 1.0)

    def op_sequence(self) -> np.ndarray:
        """Op indices: IR partitions in topological order, ops in IR order
        (the IR lists ops topologically) within each."""
        parts = self.ir.ops["part"].astype(np.int64)
        return np.concatenate([np.nonzero(parts == p)[0] for p in self.order]).astype(np.int64)

    # line 8: the partitioner the weights parameterise
    def propose(self, w: np.ndarray | None = None) -> np.ndarray:
        """split=False: the new partition id of every IR partition;
        split=True: the task id of every op."""
        w = self.candidate if w is None else w
        if self.split:
            seq = self.op_sequence()
            ow = self.op_weights(w)[seq]
            cum = np.cumsum(ow) - ow          # weight before each op
            cap = ow.sum() / max(1, self.n_tasks)
            t = np.minimum((cum / cap).astype(np.int64), self.n_tasks - 1)
            task = np.zeros(self.ir.n_ops, np.int64)
            task[seq] = t
            return task
        ws = self.weight_sum(w)
        cap = ws.sum() / max(1, self.n_tasks)
        task = np.zeros(len(ws), np.int64)
        cur, acc = 0, 0.0
        for p in self.order:
            if acc > 0 and acc + ws[p] > cap * 1.000001 and cur + 1 < self.n_tasks:
                cur += 1
                acc = 0.0
            task[p] = cur
            acc += ws[p]
        return task

    # lines 11 / 18
    def update_weights(self):
        self.weights = self.candidate.copy()


def apply(ir, task: np.ndarray):
    """The IR with every op moved to its task (same semantics): `task` maps
    IR partitions (merge proposals) or ops (split proposals) to tasks."""
    ops = ir.ops.copy()
    if len(task) == ir.n_ops and len(task) != int(ir.n_partitions):
        t = np.asarray(task, np.int64)
    else:
        t = task[ops["part"].astype(np.int64)]
    # renumber the used tasks densely, in order
    used, t = np.unique(t, return_inverse=True)
    ops["part"] = t.astype(ops["part"].dtype)
    return dataclasses.replace(ir, ops=ops, n_partitions=int(len(used)))


def accept_rate(cost: float, cur_cost: float, beta: float) -> float:
    """Eq 3: min(1, p(G*) / p(G)) = min(1, exp(beta (cost(G) - cost(G*))))."""
    if math.isinf(cur_cost):
        return 1.0
    return min(1.0, math.exp(beta * (cur_cost - cost)))


def mcmc_partition(ir, estimate_cost: Callable[[object], float], n_tasks: int, max_iter: int = 150,
                   max_unimproved: int = 30, beta: float = 1.0, seed: int = 0, log=None, split: bool = False):
    """Algorithm 1. estimate_cost(ir_candidate) -> cost (e.g. ms).
    Returns (best_ir, best_cost, history); history rows are
    (iter, cost, accepted, cur_cost), row 0 being the all-ones weights."""
    opt = Optimizer(ir, n_tasks=n_tasks, seed=seed, split=split)   # lines 3-5
    rng = random.Random(seed ^ 0x5A5A)
    # reference point (not part of Algorithm 1): the initial, all-ones weights
    cand = apply(ir, opt.propose(opt.weights))
    best = (cand, float(estimate_cost(cand)))
    hist = [(0, best[1], False, math.inf)]
    cur_cost = math.inf                          # line 1
    it = cnt = 0                                 # line 2
    while cnt < max_unimproved and it < max_iter:   # line 6
        it += 1
        opt.random_increase()                    # line 7
        task = opt.propose()                     # line 8
        cand = apply(ir, task)
        cost = float(estimate_cost(cand))        # line 9
        accepted = False
        if cur_cost > cost:                      # lines 10-14
            opt.update_weights()
            cur_cost = cost
            cnt = 0
            accepted = True
        else:                                    # lines 15-22
            if accept_rate(cost, cur_cost, beta) > rng.random():
                opt.update_weights()
                cur_cost = cost
                accepted = True
            cnt += 1
        if cost < best[1]:
            best = (cand, cost)
        hist.append((it, cost, accepted, cur_cost))
        if log:
            log(f"iter {it}: cost {cost:.4f} {'accepted' if accepted else 'rejected'} (current {cur_cost:.4f})")
    return best[0], best[1], hist


def gpu_estimator(n_stim: int = 256, cycles: int = 16, flags: int | None = None, seed: int = 0x5354494D00000000):
    """The estimator of P:L731-737: load (JIT compile) + run `cycles` cycles of
    `n_stim` seeded stimuli on the GPU; cost = evaluator ms per cycle."""
    import torch
    from rtlgen import stim
    from . import rtlsim as R
    fl = (R.F_JIT if flags is None else flags) | R.F_TIMING

    def est(ir):
        s = torch.cuda.Stream()
        sim = R.Simulator(ir, stream=s.cuda_stream, chunk_cycles=cycles, flags=fl)
        d = stim.stimulus_torch(ir, seed, 0, n_stim, 0, 2 * cycles)
        out = torch.empty((n_stim, cycles, ir.OW), dtype=torch.int32, device="cuda")
        sim.bind_device(d, n_stim, 2 * cycles)
        sim.run_device(cycles, out)          # warm-up
        sim.sync()
        a = sim.stats()
        sim.run_device(cycles, out)
        sim.sync()
        b = sim.stats()
        return (b["eval_ms"] - a["eval_ms"]) / cycles
    return est
