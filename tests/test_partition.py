"""GPU-aware MCMC partitioning (§3.2.1, Algorithm 1, Eq 1-3) — host
logic: Eq 1 weight sums, the merge-based proposal, Eq 3 acceptance, the
Algorithm 1 loop with a deterministic stand-in estimator, and that every
proposal is a valid IR the C-ABI compiler accepts."""
import math

import numpy as np
import pytest

from rtlgen import designs, shaped
from paper_conf_icpp_linrzkh22_b200 import partition as MP


def test_eq1_weight_sum_counts_top_types():
    ir = shaped.generate(3, scale=0.25)
    opt = MP.Optimizer(ir, n_tasks=4, k=30)
    assert len(opt.T) == min(30, len(np.unique(MP.node_types(ir))))
    # all-ones weights: weight_sum = ops per partition
    ws = opt.weight_sum(np.ones(len(opt.T)))
    assert np.array_equal(ws, np.bincount(ir.ops["part"], minlength=ir.n_partitions))
    # raising w_t by 1 adds N_t of the partition
    w = np.ones(len(opt.T))
    w[0] += 1
    t0 = opt.T[0]
    n_t = np.bincount(ir.ops["part"][MP.node_types(ir) == t0], minlength=ir.n_partitions)
    assert np.array_equal(opt.weight_sum(w) - ws, n_t)


def test_proposal_is_a_valid_merge():
    ir = shaped.generate(3, scale=0.25)
    opt = MP.Optimizer(ir, n_tasks=3)
    task = opt.propose(opt.weights)
    assert task.max() + 1 <= 3
    # consecutive in the partition topological order, non-decreasing
    seq = [task[p] for p in opt.order]
    assert seq == sorted(seq)
    new = MP.apply(ir, task)
    assert new.n_partitions == task.max() + 1
    assert np.array_equal(new.ops["dst"], ir.ops["dst"])          # same ops
    MP.partition_order(new)                                        # acyclic
    from paper_conf_icpp_linrzkh22_b200 import rtlsim as R
    st = R.Simulator(new, flags=R.F_HOST_ONLY).stats()
    assert st["n_partitions"] == new.n_partitions and st["n_ops"] == ir.n_ops


def _uneven(seed, n_ops=3000, P=24):
    """A random DAG cut into P bands of uneven size along its topological
    op order (an acyclic partition DAG whose tasks differ in composition)."""
    import dataclasses
    ir = designs.random_dag(seed, n_ops=n_ops, n_regs=100, n_partitions=1)
    rng = np.random.default_rng(seed)
    cuts = np.sort(rng.choice(np.arange(1, n_ops), size=P - 1, replace=False))
    ops = ir.ops.copy()
    ops["part"] = np.searchsorted(cuts, np.arange(n_ops), side="right")
    return dataclasses.replace(ir, ops=ops, n_partitions=P)


def test_weights_move_task_boundaries():
    ir = _uneven(42)
    opt = MP.Optimizer(ir, n_tasks=7)
    base = opt.propose(opt.weights)
    moved = 0
    for j in range(len(opt.T)):
        w = opt.weights.copy()
        w[j] += 5
        moved += not np.array_equal(opt.propose(w), base)
    assert moved > 0


def test_eq3_acceptance():
    assert MP.accept_rate(1.0, 2.0, beta=3.0) == 1.0                 # cheaper: always
    assert MP.accept_rate(2.0, 1.0, beta=3.0) == pytest.approx(math.exp(-3.0))
    assert MP.accept_rate(5.0, math.inf, beta=1.0) == 1.0


def test_algorithm1_loop_with_stand_in_estimator():
    """cost = |tasks - 4| + spread of task sizes: the loop accepts cheaper
    graphs, stops after max_unimproved, and returns the best it saw."""
    ir = _uneven(43, n_ops=2000, P=16)
    def est(c):
        sizes = np.bincount(c.ops["part"])
        return abs(len(sizes) - 4) + sizes.std() / sizes.mean()
    best, cost, hist = MP.mcmc_partition(ir, est, n_tasks=4, max_iter=40, max_unimproved=8, beta=50.0, seed=3)
    assert cost == min(h[1] for h in hist) and est(best) == pytest.approx(cost)
    assert len(hist) <= 41
    it_costs = [h for h in hist[1:]]
    assert any(h[2] for h in it_costs)           # the first proposal is always accepted (cur = inf)
    assert it_costs[0][2]
    # unimproved counter: the loop ends either at max_iter or after 8 non-improving iterations
    assert len(it_costs) == 40 or sum(1 for h in it_costs[-8:] if h[1] >= h[3] or not h[2]) >= 1


def test_split_proposal_chunks_the_op_sequence():
    """split=True: tasks are contiguous chunks of the partitions' topological
    op sequence, so n_tasks above the IR's partition count splits partitions
    and the task DAG stays acyclic; the compiler accepts it, the oracle's
    results do not change (partitions only change the schedule)."""
    import oracle
    from rtlgen import stim
    ir = shaped.generate(3, scale=0.1)
    opt = MP.Optimizer(ir, n_tasks=3 * ir.n_partitions, split=True)
    task = opt.propose(opt.weights)
    seq = opt.op_sequence()
    assert sorted(seq.tolist()) == list(range(ir.n_ops))
    assert np.all(np.diff(task[seq]) >= 0)                       # contiguous, in order
    new = MP.apply(ir, task)
    assert new.n_partitions > ir.n_partitions                    # partitions were split
    MP.partition_order(new)                                        # acyclic
    # raising a weight moves the cuts
    w = opt.weights.copy()
    w[0] += 5
    assert not np.array_equal(opt.propose(w), task)
    from paper_conf_icpp_linrzkh22_b200 import rtlsim as R
    assert R.Simulator(new, flags=R.F_HOST_ONLY | R.F_JIT).stats()["n_partitions"] == new.n_partitions
    st = stim.stimulus(ir, 5, np.arange(8), 0, 6)
    a, b = oracle.simulate(ir, st, digest=True), oracle.simulate(new, st, digest=True)
    assert np.array_equal(a["digest"], b["digest"])
