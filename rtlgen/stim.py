"""Counter-based seeded stimulus generator (input plumbing, no method arithmetic).

SURVEY §8(d): value(seed, s, c, k) = mix(seed + gamma * ((s * T_max + c) * IW + k)),
masked to the word's input width; mix = splitmix64 finalizer, gamma =
0x9E3779B97F4A7C15, T_max = 2^32. Any (stimulus, cycle) window can be produced
independently, so shards and parity samples need no coordination and stimulus
s is identical in every config that shares a seed.

Two implementations of the same formula: numpy (host, tests, oracle inputs) and
torch (device-side generation for the benchmark); a CPU test checks they agree.
"""
from __future__ import annotations

import numpy as np

from . import ir as I

GAMMA = 0x9E3779B97F4A7C15
T_MAX_LOG2 = 32
M1 = 0xBF58476D1CE4E5B9
M2 = 0x94D049BB133111EB

DESIGN_SEED_BASE = 0x52544C0000000000
STIM_SEED_BASE = 0x5354494D00000000
SAMPLE_SEED = 0x53414D5000000000


def _mix_np(z: np.ndarray) -> np.ndarray:
    z = z ^ (z >> np.uint64(30))
    z = z * np.uint64(M1)
    z = z ^ (z >> np.uint64(27))
    z = z * np.uint64(M2)
    return z ^ (z >> np.uint64(31))


def raw_words(seed: int, stim_idx, c0: int, nc: int, iw: int) -> np.ndarray:
    """[len(stim_idx)][nc][iw] u32 raw (unmasked) stimulus words."""
    s = np.asarray(stim_idx, dtype=np.uint64).reshape(-1, 1, 1)
    c = (np.uint64(c0) + np.arange(nc, dtype=np.uint64)).reshape(1, -1, 1)
    k = np.arange(iw, dtype=np.uint64).reshape(1, 1, -1)
    with np.errstate(over="ignore"):
        ctr = ((s << np.uint64(T_MAX_LOG2)) + c) * np.uint64(iw) + k
        z = np.uint64(seed) + np.uint64(GAMMA) * ctr
        return (_mix_np(z) & np.uint64(0xFFFFFFFF)).astype(np.uint32)


def stimulus(ir: I.IR, seed: int, stim_idx, c0: int, nc: int, mask: bool = True) -> np.ndarray:
    """Uniform random stimulus for any design: [len(stim_idx)][nc][IW] u32."""
    w = raw_words(seed, stim_idx, c0, nc, max(ir.IW, 0))
    if mask and ir.IW:
        w &= ir.input_word_masks()[None, None, :]
    return w


def tiny_stimulus(seed: int, stim_idx, T: int, c0: int = 0, nc: int | None = None,
                  mode: str = "B") -> np.ndarray:
    """Config 1 stimulus: inputs (rst, en, op, a, b).

    Mode A: free-run (rst=0, en=1). Mode B: rst/en uniform random per cycle
    with P(rst)=1/16. In both modes (a, b, op) at (s, c) is the enumeration
    index e = (s*T + c) mod 2048 (op = e[2:0], a = e[6:3], b = e[10:7]) so
    every ALU combination appears.
    """
    nc = T - c0 if nc is None else nc
    s = np.asarray(stim_idx, dtype=np.int64).reshape(-1, 1)
    c = (c0 + np.arange(nc, dtype=np.int64)).reshape(1, -1)
    e = (s * T + c) % 2048
    r = raw_words(seed, stim_idx, c0, nc, 2)
    if mode == "A":
        rst = np.zeros_like(e)
        en = np.ones_like(e)
    else:
        rst = ((r[..., 0] & 15) == 0).astype(np.int64)
        en = (r[..., 1] & 1).astype(np.int64)
    out = np.stack([rst, en, e & 7, (e >> 3) & 15, (e >> 7) & 15], axis=-1)
    return out.astype(np.uint32)


# ------------------------------------------------------------ torch version --
def stimulus_torch(ir: I.IR, seed: int, s0: int, n: int, c0: int, nc: int, device="cuda",
                   mask: bool = True):
    """Same values as :func:`stimulus` for stimuli s0..s0+n-1, as a torch int32
    tensor [n][nc][IW] on ``device`` (bit pattern of the u32 words)."""
    import torch

    def u64(x):  # python int -> int64 with the same bit pattern
        x &= (1 << 64) - 1
        return x - (1 << 64) if x >= (1 << 63) else x

    def srl(z, k):  # logical right shift on int64
        return (z >> k) & ((1 << (64 - k)) - 1)

    iw = ir.IW
    s = torch.arange(s0, s0 + n, dtype=torch.int64, device=device).view(-1, 1, 1)
    c = torch.arange(c0, c0 + nc, dtype=torch.int64, device=device).view(1, -1, 1)
    k = torch.arange(iw, dtype=torch.int64, device=device).view(1, 1, -1)
    ctr = ((s << T_MAX_LOG2) + c) * iw + k
    z = u64(seed) + u64(GAMMA) * ctr
    z = z ^ srl(z, 30)
    z = z * u64(M1)
    z = z ^ srl(z, 27)
    z = z * u64(M2)
    z = z ^ srl(z, 31)
    w = z & 0xFFFFFFFF
    if mask and iw:
        m = torch.as_tensor(ir.input_word_masks().astype(np.int64), device=device)
        w = w & m.view(1, 1, -1)
    w = torch.where(w >= (1 << 31), w - (1 << 32), w)
    return w.to(torch.int32)


def parity_sample(N: int, n: int, boundaries=(), seed: int = SAMPLE_SEED) -> np.ndarray:
    """Deterministic parity sample of ``n`` stimulus indices in [0, N)
    (SURVEY §8(c) parity policy): the warp/tile edges 0, 1, 31, 32, 33, 63,
    64, 127, 128, 255, 256, 1023, 1024, N/2 +- 1 and N-2, N-1, every multiple
    of each given boundary (shard / pipeline-chunk size) +- 1, then seeded
    uniform indices until ``n`` distinct ones (all of [0, N) when n >= N).
    Input plumbing only: shared by tools/make_golden.py and the GPU tests."""
    if n >= N:
        return np.arange(N, dtype=np.int64)
    idx = {0, 1, 31, 32, 33, 63, 64, 127, 128, 255, 256, 1023, 1024,
           N // 2 - 1, N // 2, N // 2 + 1, N - 2, N - 1}
    for b in boundaries:
        for m in range(b, N, b):
            idx |= {m - 1, m, m + 1}
    idx = {i for i in idx if 0 <= i < N}
    rng = np.random.default_rng(seed & 0xFFFFFFFF)
    while len(idx) < n:
        idx |= set(int(x) for x in rng.integers(0, N, size=n - len(idx)))
    return np.array(sorted(idx), dtype=np.int64)
