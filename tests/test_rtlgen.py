"""Input plumbing: generators are seeded, well-formed and mirror the interface."""
import os
import re

import numpy as np
import pytest

from rtlgen import designs, shaped, stim
from rtlgen import ir as I

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


def test_stimulus_counter_based_windows():
    d = designs.random_dag(1, n_ops=10, input_widths=(7, 40, 1))
    full = stim.stimulus(d, 123, np.arange(10), 0, 20)
    part = stim.stimulus(d, 123, [3, 7], 5, 10)
    assert np.array_equal(part, full[[3, 7], 5:15])
    assert np.all(full[..., 0] < 128) and np.all(full[..., 3] < 2)


def test_stimulus_torch_matches_numpy():
    torch = pytest.importorskip("torch")
    d = designs.random_dag(2, n_ops=10, input_widths=(7, 40, 1, 32))
    a = stim.stimulus(d, stim.STIM_SEED_BASE + 4, np.arange(100, 140), 3, 9)
    b = stim.stimulus_torch(d, stim.STIM_SEED_BASE + 4, 100, 40, 3, 9, device="cpu")
    assert np.array_equal(a, b.numpy().view(np.uint32))
    del torch


@pytest.mark.parametrize("cid,scale", [(2, 1.0), (3, 0.2), (4, 0.01)])
def test_shaped_designs_valid_and_seeded(oracle_lib, cid, scale):
    a = shaped.generate(cid, scale=scale)
    b = shaped.generate(cid, scale=scale)
    assert np.array_equal(a.ops, b.ops) and np.array_equal(a.width, b.width)
    oracle_lib.Design(a)          # topological order, one driver per net, widths in range
    s = a.summary()
    assert s["n_ops"] >= int(shaped.SHAPES[cid].n_ops * scale) * 0.95
    # every opcode of the mix appears
    assert len(s["opcode_hist"]) == len(I.VALUE_OPS)


def test_opcode_numbering_mirrored():
    """rtlgen/ir.py, include/rtlsim.h and oracle/oracle.h number opcodes alike."""
    h = open(os.path.join(ROOT, "include", "rtlsim.h")).read()
    o = open(os.path.join(ROOT, "oracle", "oracle.h")).read()
    for name, code in I.OPCODES.items():
        assert re.search(rf"RTLSIM_OP_{name}\s*=\s*{code}\b", h), name
        assert re.search(rf"ORC_{name}\s*=\s*{code}\b", o), name
