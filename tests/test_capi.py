"""The C-ABI library on the CPU build host: it loads, exports every symbol
include/rtlsim.h declares, and its host-side compiler (validation, levelizer,
layout, byte accounting) behaves — no compute calls without a GPU."""
import ctypes
import os
import re

import numpy as np
import pytest

from rtlgen import designs, shaped
from rtlgen import ir as I
from rtlgen.builder import Builder

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))


@pytest.fixture(scope="module")
def R():
    from paper_conf_icpp_linrzkh22_b200 import build, rtlsim
    build.build()
    return rtlsim


def test_exports_every_declared_symbol(R):
    hdr = open(os.path.join(ROOT, "include", "rtlsim.h")).read()
    declared = set(re.findall(r"\b(rtlsim_[a-z_]+)\s*\(", hdr))
    declared -= {"rtlsim_producer", "rtlsim_consumer"}
    assert {"rtlsim_load", "rtlsim_bind", "rtlsim_run"} <= declared
    lib = ctypes.CDLL(R.LIB_PATH)
    for name in sorted(declared):
        assert hasattr(lib, name), name
    assert declared == set(R.EXPORTS)


def _load(R, ir, **kw):
    return R.Simulator(ir, flags=R.F_HOST_ONLY, **kw)


def test_host_only_compile_and_stats(R):
    ir = designs.tiny_dut()
    st = _load(R, ir).stats()
    assert st["n_ops"] == ir.n_ops and st["iw"] == 5 and st["ow"] == ir.OW and st["rw"] == ir.RW
    # B_floor = sum_regs 2 b(w) + sum_in b(w) + sum_out b(w), b = 1/8, 1, 2, 4*ceil(w/32)
    b = lambda w: 0.125 if w == 1 else 1 if w <= 8 else 2 if w <= 16 else 4 * ((w + 31) // 32)
    want = (sum(2 * b(int(ir.width[q])) for q in ir.reg_q) + sum(b(int(ir.width[s])) for s in ir.input_sig)
            + sum(b(int(ir.width[s])) for s in ir.output_sig))
    assert st["b_floor"] == pytest.approx(want)
    assert st["n_steps"] >= 3 and st["smem_words"] > 0


def _live_ops_reference(ir):
    """Ops whose value reaches a register D or an output (reverse reachability
    over the op DAG, written independently of csrc/compile.cpp)."""
    import numpy as np
    from rtlgen import ir as I
    op = ir.ops
    drv = {int(d): i for i, d in enumerate(op["dst"])}
    need = set(int(s) for s in ir.reg_d) | set(int(s) for s in ir.output_sig)
    stack, live = list(need), set()
    while stack:
        s = stack.pop()
        i = drv.get(s)
        if i is None or i in live:
            continue
        live.add(i)
        for f in ("a", "b", "c"):
            v = int(op[f][i])
            if v != 0xFFFFFFFF and v not in need:
                need.add(v)
                stack.append(v)
    return len(live)


@pytest.mark.parametrize("cid", [2, 3])
def test_dead_logic_elimination_counts(R, cid):
    """Only ops that can reach an observable (register D / output) are
    scheduled; RTLSIM_F_NO_DCE schedules all of them."""
    ir = shaped.generate(cid)
    st = _load(R, ir).stats()
    assert st["n_ops"] == ir.n_ops
    assert st["n_live_ops"] == _live_ops_reference(ir) < ir.n_ops
    full = R.Simulator(ir, flags=R.F_HOST_ONLY | R.F_NO_DCE).stats()
    assert full["n_live_ops"] == ir.n_ops and full["word_ops"] == st["word_ops"]
    assert st["live_word_ops"] < full["live_word_ops"] and st["n_desc"] < full["n_desc"]


def test_partitioned_design_uses_cross_partition_nets(R):
    ir = designs.random_dag(5, n_ops=200, n_regs=10, n_partitions=3)
    st = _load(R, ir).stats()
    assert st["b_part"] > 0 and st["xrows_bit"] + st["xrows_u8"] + st["xrows_u16"] + st["xrows_u32"] > 0


def test_shaped_configs_fit_shared_memory(R):
    for cid in (2, 3):
        st = _load(R, shaped.generate(cid)).stats()
        assert st["smem_words"] * 4 <= 227 * 1024, (cid, st["smem_words"])
        assert st["op_lanes"] >= 1


def test_smem_budget_spills_and_narrows(R):
    """A budget below the working set: the schedule is narrowed (more steps),
    long-lived values spill to extra cross-partition rows, the slot area fits,
    and the spill traffic is accounted in b_state."""
    ir = shaped.generate(3, scale=0.25)
    free = R.Simulator(ir, flags=R.F_HOST_ONLY, op_lanes=2).stats()
    lim = 13000
    st = R.Simulator(ir, flags=R.F_HOST_ONLY, op_lanes=2, smem_limit=lim).stats()
    assert free["smem_words"] * 4 > lim and free["b_spill"] == 0
    assert st["smem_words"] * 4 <= lim and st["b_spill"] > 0
    assert st["n_steps"] > free["n_steps"]
    assert st["b_state"] == pytest.approx(free["b_state"] + st["b_spill"])
    xr = lambda s: s["xrows_bit"] + s["xrows_u8"] + s["xrows_u16"] + s["xrows_u32"]
    assert xr(st) > xr(free)
    with pytest.raises(R.RtlsimError) as e:     # below the unspillable floor
        R.Simulator(ir, flags=R.F_HOST_ONLY, op_lanes=2, smem_limit=2048)
    assert e.value.code == -5


def _expect_error(R, ir, code):
    with pytest.raises(R.RtlsimError) as e:
        _load(R, ir)
    assert e.value.code == code, (e.value, code)


def test_validation_errors(R):
    # comb loop
    b = Builder()
    x = b.input(4)
    y = b.op("NOT", 4, x)
    z = b.op("NOT", 4, y)
    ir = b.build()
    ir.ops["a"][0] = z          # y = ~z, z = ~y
    _expect_error(R, ir, -3)
    # double driver
    b = Builder()
    x = b.input(4)
    y = b.op("NOT", 4, x)
    ir = b.build()
    ir.ops = np.concatenate([ir.ops, ir.ops])
    _expect_error(R, ir, -2)
    # width 0 / > 1024
    ir = designs.listing2_dut()
    ir.width[0] = 0
    _expect_error(R, ir, -2)
    ir = designs.listing2_dut()
    ir.width[0] = 1025
    _expect_error(R, ir, -2)
    # MUL wider than 64 bits
    b = Builder()
    x = b.input(65)
    b.op("MUL", 8, x, x)
    _expect_error(R, b.build(), -4)
    # SLICE out of range
    b = Builder()
    x = b.input(8)
    b.op("SLICE", 4, x, imm=5)
    _expect_error(R, b.build(), -2)
    # partition DAG cycle: p0 -> p1 -> p0
    b = Builder()
    x = b.input(4)
    b.partition(0)
    u = b.op("NOT", 4, x)
    b.partition(1)
    v = b.op("NOT", 4, u)
    b.partition(0)
    b.op("NOT", 4, v)
    _expect_error(R, b.build(), -2)
    # the last load error is reported with a message
    assert R.rtlsim_last_error(None)


def test_unordered_ops_are_sorted(R):
    """Ops may be given in any order; the levelizer sorts them."""
    ir = designs.random_dag(7, n_ops=50)
    rev = I.IR(**{f: getattr(ir, f) for f in ("width", "kind", "ops", "reg_q", "reg_d", "reg_init", "const_sig",
                                               "const_words", "input_sig", "output_sig")})
    rev.ops = ir.ops[::-1].copy()
    assert _load(R, rev).stats()["n_ops"] == 50


def test_product_does_not_import_oracle():
    pkg = os.path.join(ROOT, "paper_conf_icpp_linrzkh22_b200")
    for dirpath, _, files in os.walk(pkg):
        for f in files:
            if f.endswith((".py", ".cu", ".cpp", ".h")):
                src = open(os.path.join(dirpath, f)).read()
                assert "import oracle" not in src and "from oracle" not in src and "oracle.h" not in src, f


def test_jit_cubin_cache(R, tmp_path, monkeypatch):
    """RTLSIM_JIT_CACHE: the first load writes one cubin per partition
    module, a second load of the same design reads them back (same bytes)."""
    monkeypatch.setenv("RTLSIM_JIT_CACHE", str(tmp_path / "jc"))
    ir = designs.random_dag(5, n_ops=200, n_regs=10, n_partitions=3)
    a = R.Simulator(ir, flags=R.F_HOST_ONLY | R.F_JIT).stats()
    files = sorted(p.name for p in (tmp_path / "jc").iterdir())
    assert len(files) == 3 and all(f.endswith(".cubin") for f in files)
    b = R.Simulator(ir, flags=R.F_HOST_ONLY | R.F_JIT).stats()
    assert b["jit_cubin_bytes"] == a["jit_cubin_bytes"] > 0
    assert sorted(p.name for p in (tmp_path / "jc").iterdir()) == files


def test_jit_nspec_windows(R, tmp_path, monkeypatch):
    """N-specialised JIT code (state-row offsets as immediates from a window
    register per arena base) compiles, differs from the generic code, and
    carries the N_pad guard; the generic code keeps the run-time row stride."""
    ir = designs.random_dag(7, n_ops=300, n_regs=12, n_partitions=2)
    gen, spec = tmp_path / "g", tmp_path / "s"
    gen.mkdir()
    spec.mkdir()
    monkeypatch.setenv("RTLSIM_JIT_SAVE", str(gen))
    R.Simulator(ir, flags=R.F_HOST_ONLY | R.F_JIT)
    monkeypatch.setenv("RTLSIM_JIT_SAVE", str(spec))
    monkeypatch.setenv("RTLSIM_JIT_NSPEC", "4096")
    assert R.Simulator(ir, flags=R.F_HOST_ONLY | R.F_JIT).stats()["jit_cubin_bytes"] > 0
    g = "".join(p.read_text() for p in sorted(gen.iterdir()))
    s = "".join(p.read_text() for p in sorted(spec.iterdir()))
    assert "mad.wide.u32" in g and "%N4," in g and "trap" not in g
    assert "setp.ne.u32 %pn, %N, 4096" in s and "@%pn trap" in s
    assert "mad.wide.u32 %rd" not in s.split(".entry")[0].split("rtl_steps_0")[-1]


def test_jit_dead_store_elimination_compiles(R, tmp_path, monkeypatch):
    """RTLSIM_JIT_DSE=1 drops slot stores whose readers all take the value
    from the writer's register: fewer st.shared, the code still compiles,
    every remaining ld.shared is unchanged in number (reads are not moved)."""
    ir = designs.random_dag(11, n_ops=400, n_regs=16, n_partitions=2)
    counts = {}
    for dse in ("0", "1"):
        d = tmp_path / dse
        d.mkdir()
        monkeypatch.setenv("RTLSIM_JIT_SAVE", str(d))
        monkeypatch.setenv("RTLSIM_JIT_DSE", dse)
        assert R.Simulator(ir, flags=R.F_HOST_ONLY | R.F_JIT).stats()["jit_cubin_bytes"] > 0
        txt = "".join(p.read_text().split(".func rtl_steps_0")[-1] for p in sorted(d.iterdir()))
        counts[dse] = (txt.count("st.shared"), txt.count("ld.shared"))
    assert counts["1"][0] < counts["0"][0]
    assert counts["1"][1] == counts["0"][1]


def test_memory_validation_host_only(R):
    """Memories (reading 12) through the C ABI on the host: accepted with the
    JIT backend, E_UNSUPPORTED without it; a MEMRD of a missing memory and an
    address wider than 32 bits are rejected."""
    ir = designs.regfile_dut()
    sim = R.Simulator(ir, flags=R.F_HOST_ONLY | R.F_JIT)
    assert sim.stats()["n_live_ops"] > 0
    with pytest.raises(R.RtlsimError) as ei:
        R.Simulator(ir, flags=R.F_HOST_ONLY)
    assert ei.value.code == -4
    bad = designs.mem_seq_dut()
    bad.ops["imm"][bad.ops["opcode"] == I.OPCODES["MEMRD"]] = 3
    with pytest.raises(R.RtlsimError) as ei:
        R.Simulator(bad, flags=R.F_HOST_ONLY | R.F_JIT)
    assert ei.value.code == -2
    b = Builder("wideaddr")
    a = b.input(40)
    m = b.mem(8, 4)
    b.output(b.memrd(m, a))
    with pytest.raises(R.RtlsimError) as ei:
        R.Simulator(b.build(), flags=R.F_HOST_ONLY | R.F_JIT)
    assert ei.value.code == -4


def test_tmem_schedule_host_only(R, tmp_path, monkeypatch):
    """TMEM schedules compile host-only: computed U32 values
    get TMEM columns (slot = 0x8000 + 32 col), the shared-memory slot area
    shrinks, and the generated PTX allocates / frees TMEM and moves values
    with tcgen05.ld / tcgen05.st under the step-barrier fences."""
    ir = designs.random_dag(502, n_ops=300, n_regs=24, n_partitions=3, input_widths=(7, 33, 1, 64, 100),
                            max_width=1024)
    monkeypatch.setenv("RTLSIM_JIT_CACHE", "")
    monkeypatch.setenv("RTLSIM_JIT_SAVE", str(tmp_path))
    monkeypatch.setenv("RTLSIM_JIT_TMEM", "0")
    classic = R.Simulator(ir, flags=R.F_HOST_ONLY | R.F_JIT).stats()
    monkeypatch.setenv("RTLSIM_JIT_TMEM", "1")
    st = R.Simulator(ir, flags=R.F_HOST_ONLY | R.F_JIT).stats()
    assert classic["tmem_cols"] == 0 and 0 < st["tmem_cols"] <= 512
    assert st["smem_words"] < classic["smem_words"]
    assert st["op_lanes"] <= 8 and st["jit_sass_instructions"] > 0
    ptx = "".join(p.read_text() for p in tmp_path.glob("part*.ptx"))
    for needle in ("tcgen05.alloc", "tcgen05.dealloc", "tcgen05.ld.sync.aligned.32x32b", "tcgen05.st.sync.aligned.32x32b",
                   "tcgen05.wait::st", "tcgen05.fence::before_thread_sync", "tcgen05.fence::after_thread_sync"):
        assert needle in ptx, needle
