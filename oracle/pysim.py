"""Pure-Python cycle loop over :mod:`oracle.ops_ref` — small cases only.

TEST INFRASTRUCTURE ONLY. Listing 1 for one stimulus:
inputs, then every op in order, then pre-edge outputs, then all registers at
once. Used to pin the C oracle on random DAGs (brute force on tiny inputs).
"""
from __future__ import annotations

import numpy as np

from rtlgen import ir as I

from . import ops_ref


def _val(ws, w):
    return I.words_to_int(ws) & ops_ref.mask(w)


def simulate(ir: I.IR, stim: np.ndarray, regs_in=None):
    """stim [N][T][IW] -> (out [N][T][OW], regs [N][RW]) as numpy u32 arrays."""
    N, T = stim.shape[0], stim.shape[1]
    width = [int(x) for x in ir.width]
    outs = np.zeros((N, T, ir.OW), np.uint32)
    regs = np.zeros((N, ir.RW), np.uint32)
    consts = {}
    k = 0
    for s in ir.const_sig:
        n = I.nwords(width[s])
        consts[int(s)] = _val(ir.const_words[k:k + n], width[s])
        k += n
    init = []
    k = 0
    for q in ir.reg_q:
        n = I.nwords(width[q])
        init.append(_val(ir.reg_init[k:k + n], width[q]))
        k += n
    ops = [(I.OPNAMES[int(o["opcode"])], int(o["dst"]), int(o["a"]), int(o["b"]), int(o["c"]),
            int(o["imm"])) for o in ir.ops]
    # memories (reading 12): entry lists, read by MEMRD, written at
    # the clock edge by the ports in order
    n_mems = getattr(ir, "n_mems", 0)
    mem_init, k = [], 0
    for m in range(n_mems):
        wm, dm = int(ir.mem_width[m]), int(ir.mem_depth[m])
        n = I.nwords(wm)
        mem_init.append([_val(ir.mem_init[k + n * e:k + n * (e + 1)], wm) for e in range(dm)])
        k += n * dm
    mems_out = []
    for s in range(N):
        M = [list(x) for x in mem_init]
        if regs_in is None:
            R = list(init)
        else:
            R, k = [], 0
            for q in ir.reg_q:
                n = I.nwords(width[q])
                R.append(_val(regs_in[s][k:k + n], width[q]))
                k += n
        for c in range(T):
            V = dict(consts)
            k = 0
            for i in ir.input_sig:
                n = I.nwords(width[i])
                V[int(i)] = _val(stim[s, c, k:k + n], width[i])
                k += n
            for q, v in zip(ir.reg_q, R):
                V[int(q)] = v
            for name, d, a, b, cc, imm in ops:
                if name == "MEMRD":
                    V[d] = M[imm][V[a]] if V[a] < len(M[imm]) else 0
                    continue
                V[d] = ops_ref.evaluate(
                    name, width[d], V[a], width[a],
                    V.get(b, 0) if b != I.NONE else 0, width[b] if b != I.NONE else 0,
                    V.get(cc, 0) if cc != I.NONE else 0, width[cc] if cc != I.NONE else 0, imm)
            row = []
            for o in ir.output_sig:
                row += I.int_to_words(V[int(o)], width[o])
            outs[s, c] = row
            R = [V[int(d)] & ops_ref.mask(width[q]) for q, d in zip(ir.reg_q, ir.reg_d)]
            for m, a, dd, en in (ir.mem_wport if n_mems else []):
                m, a, dd, en = int(m), int(a), int(dd), int(en)
                if V[en] != 0 and V[a] < len(M[m]):
                    M[m][V[a]] = V[dd] & ops_ref.mask(int(ir.mem_width[m]))
        mems_out.append([w for m in range(n_mems) for v in M[m]
                         for w in I.int_to_words(v, int(ir.mem_width[m]))])
        row = []
        for q, v in zip(ir.reg_q, R):
            row += I.int_to_words(v, width[q])
        regs[s] = row
    if n_mems:
        return outs, regs, np.asarray(mems_out, np.uint32).reshape(N, -1)
    return outs, regs
