"""Golden parity digests for the full-size configs, computed by the CPU
oracle ONLY (oracle/ + rtlgen/ input plumbing; nothing from the CUDA path).

For each sampled stimulus s of a config (rtlgen.stim.parity_sample) the oracle
simulates ALL T cycles of BASELINE.json's configuration and this script stores

  * sha256 of digest[s][0..T-1] (the per-cycle DIGEST of DESIGN.md §3 over
    every output word and every next-state register word, as little-endian
    u64), and
  * sha256 of the final register words regs[s][0..RW-1] (little-endian u32;
    configs 2-3 only: at config 4 the GPU side would have to export 49 GB of
    registers, and the last cycle's digest already folds in every register).

The GPU tests (tests/test_gpu_golden.py) run the same N x T on the device and
compare the same hashes ("all signal outputs match the
golden reference"). Resumable: lines already written are kept.

  python tools/make_golden.py 3 [--threads 6]
"""
import argparse
import hashlib
import os
import sys
import time

import numpy as np

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
sys.path.insert(0, ROOT)

import oracle  # noqa: E402
from rtlgen import shaped, stim  # noqa: E402

# config: (N, T, sample size, boundaries, hash final registers)
CONFIGS = {
    2: (4096, 10000, 1024, (1024,), True),   # 1024 of 4096: ~1 h of oracle time on the 8-core build host (4096 would be ~3.5 h)
    3: (16384, 10000, 1024, (4096,), True),
    4: (65536, 1000, 1024, (8192,), False),
    5: (262144, 1000, 256, (32768,), False),
}


def path(cid):
    return os.path.join(ROOT, "tests", "golden", f"config{cid}.txt")


def header(cid):
    N, T, n, b, rh = CONFIGS[cid]
    d = 4 if cid == 5 else cid
    return [f"# golden per-stimulus hashes, config {cid}: N={N} T={T} sample={n} boundaries={list(b)}",
            f"# design seed {stim.DESIGN_SEED_BASE + d:#x} (rtlgen.shaped.generate({d})), "
            f"stimulus seed {stim.STIM_SEED_BASE + d:#x}, sample seed {stim.SAMPLE_SEED:#x}",
            "# written by tools/make_golden.py from oracle/ only (PAPER.md P:L1128-1129)",
            "# columns: stimulus sha256(digest[s][0..T-1] u64 LE)[:32] sha256(regs[s] u32 LE)[:32] or -"]


def read(cid):
    """{stimulus: (digest_hash, regs_hash or None)}"""
    res = {}
    p = path(cid)
    if not os.path.exists(p):
        return res
    for line in open(p):
        if line.startswith("#") or not line.strip():
            continue
        parts = line.split()
        if len(parts) != 3 or len(parts[1]) != 32:   # a line cut short by a killed run
            continue
        s, dh, rh = parts
        res[int(s)] = (dh, None if rh == "-" else rh)
    return res


def sample(cid):
    N, T, n, b, _ = CONFIGS[cid]
    return stim.parity_sample(N, n, b)


def main():
    ap = argparse.ArgumentParser()
    ap.add_argument("config", type=int, choices=sorted(CONFIGS))
    ap.add_argument("--threads", type=int, default=6)
    ap.add_argument("--block", type=int, default=48)
    ap.add_argument("--reverse", action="store_true", help="work from the end of the sample (a second host)")
    ap.add_argument("--out", default=None, help="append to this file instead (merged into tests/golden later)")
    ap.add_argument("--limit", type=int, default=0, help="stop after this many stimuli")
    a = ap.parse_args()
    cid = a.config
    N, T, n, b, want_regs = CONFIGS[cid]
    d = 4 if cid == 5 else cid
    ir = shaped.generate(d)
    D = oracle.Design(ir)
    seed = stim.STIM_SEED_BASE + d
    idx = sample(cid)
    done = read(cid)
    todo = [int(i) for i in idx if int(i) not in done]
    if a.reverse:
        todo = todo[::-1]
    if a.limit:
        todo = todo[:a.limit]
    p = a.out or path(cid)
    if not os.path.exists(p):
        with open(p, "w") as f:
            f.write("\n".join(header(cid)) + "\n")
    t0 = time.time()
    for k in range(0, len(todo), a.block):
        blk = np.array(todo[k:k + a.block], dtype=np.int64)
        st = stim.stimulus(ir, seed, blk, 0, T)
        r = D.simulate(st, out=False, regs=True, digest=True, threads=a.threads)
        lines = []
        for j, s in enumerate(blk):
            dh = hashlib.sha256(np.ascontiguousarray(r["digest"][j], "<u8").tobytes()).hexdigest()[:32]
            rh = hashlib.sha256(np.ascontiguousarray(r["regs"][j], "<u4").tobytes()).hexdigest()[:32] \
                if want_regs else "-"
            lines.append(f"{int(s)} {dh} {rh}\n")
        with open(p, "a") as f:   # one write per block, flushed at once
            f.write("".join(lines))
        el = time.time() - t0
        print(f"config {cid}: {k + len(blk)}/{len(todo)} stimuli, {el:.0f} s", flush=True)


if __name__ == "__main__":
    main()
