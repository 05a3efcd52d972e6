"""Instruction-fetch microbenchmark (sm_100a): how fast can an SM issue
straight-line code that does not fit its instruction caches, as a function of
how many warps share each code stream?

One CTA of W warps per SM (grid = #SMs); warp w runs code copy w % K (K
distinct copies of M straight-line integer instructions, 8 independent
chains: LOP3 / IADD3 mix, nothing foldable). Reported: warp-instructions
issued per SM per cycle (IPC) and code bytes fetched per SM per cycle.
A control runs one copy R times in a loop (the code stays cached).

python tools/fetch_bench.py   (needs a GPU; used for DESIGN.md §5.2)
"""
import json
import os
import subprocess
import sys
import tempfile

import numpy as np


def ptx(K, M, loop=1, group=1):
    s = [".version 8.8", ".target sm_100a", ".address_size 64", "",
         ".visible .entry k(.param .u64 out, .param .u32 reps)", "{",
         "\t.reg .b32 %r<16>;", "\t.reg .b32 %t, %w, %c, %rep, %nrep;", "\t.reg .b64 %a;", "\t.reg .pred %p;",
         "\tmov.u32 %t, %tid.x;", "\tshr.u32 %w, %t, 5;", f"\tdiv.u32 %w, %w, {group};", f"\trem.u32 %c, %w, {K};",
         "\tld.param.u32 %nrep, [reps];"]
    for i in range(10):
        s.append(f"\tadd.u32 %r{i}, %t, {i * 7919 + 13};")
    s.append("\tmov.u32 %rep, 0;")
    labs = [f"$C{k}" for k in range(K)]
    if K > 1:
        s.append("$T: .branchtargets " + ", ".join(labs) + ";")
        s.append("\tbrx.idx %c, $T;")
    for k in range(K):
        s.append(f"{labs[k]}:")
        if loop:
            s.append(f"$L{k}:")
        for t in range(M):
            i = (t + k) % 8
            if t % 2 == 0:
                s.append(f"\tlop3.b32 %r{i}, %r{i}, %r{(i + 3) % 8}, %r{(i + 5) % 8}, {0x96 ^ (k & 0x0F)};")
            else:
                s.append(f"\tadd.u32 %r{i}, %r{i}, %r{(i + 1) % 8};")
        if loop:
            s.append("\tadd.u32 %rep, %rep, 1;")
            s.append("\tsetp.lt.u32 %p, %rep, %nrep;")
            s.append(f"\t@%p bra.uni $L{k};")
        s.append("\tbra.uni $E;")
    s.append("$E:")
    for i in range(1, 8):
        s.append(f"\txor.b32 %r0, %r0, %r{i};")
    s += ["\t.reg .b64 %o;", "\tld.param.u64 %a, [out];", "\tcvta.to.global.u64 %a, %a;",
          "\tmul.wide.u32 %o, %t, 4;", "\tadd.u64 %a, %a, %o;", "\tst.global.u32 [%a], %r0;", "\tret;", "}"]
    return "\n".join(s) + "\n"


def main():
    from cuda.bindings import driver as cu
    import ctypes

    def ck(r):
        if isinstance(r, tuple):
            err, rest = r[0], r[1:]
        else:
            err, rest = r, ()
        assert int(err) == 0, err
        return rest[0] if len(rest) == 1 else rest
    ck(cu.cuInit(0))
    dev = ck(cu.cuDeviceGet(0))
    ctx = ck(cu.cuDevicePrimaryCtxRetain(dev))
    ck(cu.cuCtxSetCurrent(ctx))
    nsm = ck(cu.cuDeviceGetAttribute(cu.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_MULTIPROCESSOR_COUNT, dev))
    clk = ck(cu.cuDeviceGetAttribute(cu.CUdevice_attribute.CU_DEVICE_ATTRIBUTE_CLOCK_RATE, dev)) * 1e3
    out = ck(cu.cuMemAlloc(4 * 1024 * 64))
    res = []
    W = int(os.environ.get("W", 32))
    G = int(os.environ.get("GROUP", 1))   # warps w .. w+G-1 share a copy (G=4: one per SMSP)
    cases = []
    for M in (16384,):
        for K in (1, 2, 4, 8, 14, 16, 32):
            if K * G <= W:
                cases.append((K, M, 0, 1))
    cases += [(1, 1024, 1, 64), (8, 1024, 1, 64), (14, 1024, 1, 64), (32, 1024, 1, 64)]
    for K, M, loop, reps in cases:
        with tempfile.TemporaryDirectory() as d:
            p = os.path.join(d, "k.ptx")
            open(p, "w").write(ptx(K, M, loop, G))
            subprocess.run(["ptxas", "-arch=sm_100a", "-O3", p, "-o", os.path.join(d, "k.cubin")], check=True)
            data = open(os.path.join(d, "k.cubin"), "rb").read()
        mod = ck(cu.cuModuleLoadData(data))
        fn = ck(cu.cuModuleGetFunction(mod, b"k"))
        a_out = ctypes.c_uint64(int(out))
        a_reps = ctypes.c_uint32(reps)
        args = (ctypes.c_void_p * 2)(ctypes.addressof(a_out), ctypes.addressof(a_reps))
        e0, e1 = ck(cu.cuEventCreate(0)), ck(cu.cuEventCreate(0))
        for it in range(4):
            ck(cu.cuEventRecord(e0, 0))
            ck(cu.cuLaunchKernel(fn, nsm, 1, 1, 32 * W, 1, 1, 0, 0, ctypes.addressof(args), 0))
            ck(cu.cuEventRecord(e1, 0))
            ck(cu.cuEventSynchronize(e1))
        ms = ck(cu.cuEventElapsedTime(e0, e1))
        cycles = ms * 1e-3 * clk
        instr = W * (M + (3 if loop else 0)) * reps
        r = {"group": G, "K_copies": K, "M_instr": M, "loop_reps": reps, "warps_per_sm": W, "ms": ms,
             "ipc_per_sm": instr / cycles, "code_bytes_per_sm_cycle": instr / cycles * 16 / max(1, W / K) if not loop else None,
             "warps_per_stream": W / K}
        print(json.dumps(r), flush=True)
        res.append(r)
        ck(cu.cuModuleUnload(mod))


if __name__ == "__main__":
    main()
