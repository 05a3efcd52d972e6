"""Aggregate an ncu report's source page (SASS, per-PC stall samples) by
opcode: where the warps of a kernel wait, per instruction kind.

python tools/ncu_by_opcode.py <report.ncu-rep> [out.txt]
"""
import collections
import csv
import io
import subprocess
import sys


def main():
    rep = sys.argv[1]
    txt = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr_i = next(i for i, r in enumerate(rows) if r and r[0] == "Address")
    hdr = rows[hdr_i]
    stall_cols = [i for i, h in enumerate(hdr) if h.startswith("stall_") and "(Not Issued)" not in h]
    src_i, ex_i, samp_i = hdr.index("Source"), hdr.index("Instructions Executed"), hdr.index("# Samples")
    agg = collections.defaultdict(lambda: collections.Counter())
    tot = collections.Counter()
    for r in rows[hdr_i + 1:]:
        if len(r) != len(hdr):
            continue
        op = r[src_i].strip().split()
        if not op:
            continue
        k = op[0]
        if k.startswith("@"):
            k = op[1] if len(op) > 1 else k
        k = k.split(".")[0]
        c = agg[k]
        c["exec"] += int(r[ex_i] or 0)
        c["samples"] += int(r[samp_i] or 0)
        c["n_pc"] += 1
        for i in stall_cols:
            v = int(r[i] or 0)
            c[hdr[i]] += v
            tot[hdr[i]] += v
    all_s = sum(c["samples"] for c in agg.values()) or 1
    all_e = sum(c["exec"] for c in agg.values()) or 1
    lines = [f"{rep}: {all_s} samples, {all_e} warp-instructions executed",
             "totals: " + ", ".join(f"{k[6:]} {100 * v / all_s:.1f}%" for k, v in tot.most_common(8))]
    lines.append(f"{'opcode':12s} {'exec%':>6s} {'samp%':>6s}  top stalls (% of all samples)")
    for k, c in sorted(agg.items(), key=lambda kv: -kv[1]["samples"])[:25]:
        st = sorted(((v, n) for n, v in c.items() if n.startswith("stall_")), reverse=True)[:4]
        lines.append(f"{k:12s} {100 * c['exec'] / all_e:6.1f} {100 * c['samples'] / all_s:6.1f}  " +
                     ", ".join(f"{n[6:]} {100 * v / all_s:.1f}" for v, n in st if v))
    out = "\n".join(lines)
    print(out)
    if len(sys.argv) > 2:
        open(sys.argv[2], "w").write(out + "\n")


if __name__ == "__main__":
    main()
