"""Summarise an ncu report (details + raw metrics + top stall PCs) into text
and JSON under profiles/: python tools/ncu_summary.py <report.ncu-rep> <out-prefix>
[--stim-cycles K] (stimulus-cycles the profiled launch covered, for per-unit
DRAM bytes)."""
import csv
import io
import json
import subprocess
import sys

KEYS = ["Duration", "DRAM Throughput", "Memory Throughput", "Executed Ipc Active", "Issue Slots Busy",
        "Issued Instructions", "Warp Cycles Per Issued Instruction", "Eligible Warps Per Scheduler",
        "Active Warps Per Scheduler", "No Eligible", "Registers Per Thread", "Achieved Occupancy",
        "Dynamic Shared Memory Per Block", "L1/TEX Hit Rate", "L2 Hit Rate", "Mem Busy", "SM Frequency",
        "Compute (SM) Throughput", "Waves Per SM", "Block Size", "Grid Size"]
RAW = ["dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__time_duration.sum", "sm__inst_executed.sum",
       "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum", "lts__t_bytes.sum"]


def run(args):
    return subprocess.run(["ncu", "-i"] + args, capture_output=True, text=True).stdout


def main():
    rep, out = sys.argv[1], sys.argv[2]
    stim_cycles = None
    if "--stim-cycles" in sys.argv:
        stim_cycles = float(sys.argv[sys.argv.index("--stim-cycles") + 1])
    det = run([rep, "--page", "details"])
    lines = [l for l in det.splitlines() if any(k in l for k in KEYS)]
    raw = list(csv.reader(io.StringIO(run([rep, "--page", "raw", "--csv"]))))
    res = {}
    if len(raw) >= 3:
        hdr, units, vals = raw[0], raw[1], raw[2]
        for k, u, v in zip(hdr, units, vals):
            if k in RAW or k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued"):
                res[k] = {"value": v, "unit": u}
    # top stall PCs
    src = list(csv.reader(io.StringIO(run([rep, "--page", "source", "--csv", "--print-source", "sass"]))))
    top = []
    if len(src) > 2:
        h = src[1]
        iE, iS = h.index("Instructions Executed"), h.index("Warp Stall Sampling (All Samples)")
        rows = [r for r in src[2:] if r and r[0].startswith("0x")]
        base = int(rows[0][0], 16)
        tot = sum(int(r[iS] or 0) for r in rows) or 1
        for r in sorted(rows, key=lambda r: -int(r[iS] or 0))[:15]:
            top.append(f"{int(r[0], 16) - base:#07x} {int(r[iS] or 0) * 100 / tot:5.1f}% stalls "
                       f"{int(r[iE] or 0):>12d} exec  {r[1].strip()[:70]}")
    summary = {"report": rep, "details": lines, "raw": res, "top_stall_pcs": top}

    def num(key):
        v = res.get(key, {})
        try:
            x = float(v.get("value", "nan").replace(",", ""))
        except ValueError:
            return None
        u = v.get("unit", "")
        scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}.get(u, 1)
        return x * scale

    rd, wr = num("dram__bytes_read.sum"), num("dram__bytes_write.sum")
    if rd is not None and wr is not None:
        summary["dram_bytes"] = rd + wr
        if stim_cycles:
            summary["dram_bytes_per_stim_cycle"] = (rd + wr) / stim_cycles
    json.dump(summary, open(out + ".json", "w"), indent=1)
    with open(out + ".txt", "w") as f:
        f.write(f"ncu summary of {rep}\n\n")
        f.write("\n".join(lines) + "\n\nraw:\n")
        for k, v in res.items():
            f.write(f"  {k} = {v['value']} {v['unit']}\n")
        if "dram_bytes" in summary:
            f.write(f"\nDRAM bytes (read+write) = {summary['dram_bytes']:.4g}\n")
        if "dram_bytes_per_stim_cycle" in summary:
            f.write(f"DRAM bytes per stimulus-cycle = {summary['dram_bytes_per_stim_cycle']:.4g}\n")
        f.write("\ntop stall PCs:\n" + "\n".join(top) + "\n")
    print(open(out + ".txt").read())


if __name__ == "__main__":
    main()
