"""Sum ncu's per-launch DRAM bytes over the rtl_jit_part launches of one
simulated cycle into profiles/ncu_config<c>.json (bench.py's roofline
`traffic`): python tools/cycle_dram.py <launches.csv> <config> <N> <n_launches> <out.json>"""
import csv
import json
import sys

path, cid, N, nl, out = sys.argv[1], int(sys.argv[2]), int(sys.argv[3]), int(sys.argv[4]), sys.argv[5]
rows = list(csv.reader(open(path)))
hdr = None
per = {}
for r in rows:
    if "Kernel Name" in r:
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d["Kernel Name"] != "rtl_jit_part":
            continue
        v = float(d["Metric Value"].replace(",", ""))
        u = d["Metric Unit"]
        if d["Metric Name"].startswith("dram__bytes"):
            v *= {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}.get(u, 1)
        elif d["Metric Name"] == "gpu__time_duration.sum":
            v *= {"ns": 1e-6, "us": 1e-3, "ms": 1.0}.get(u, 1)
        per.setdefault(d["ID"], {})[d["Metric Name"]] = v
ids = sorted(per, key=int)[-nl:]   # the last full cycle
b = sum(per[i].get("dram__bytes_read.sum", 0) + per[i].get("dram__bytes_write.sum", 0) for i in ids)
t = sum(per[i].get("gpu__time_duration.sum", 0) for i in ids)
res = {"source": f"ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none "
                 f"over the {len(ids)} rtl_jit_part launches of one cycle, config {cid}, N={N} ({path})",
       "launches": len(ids), "dram_bytes_per_cycle": b, "dram_bytes_per_stim_cycle": b / N,
       "kernel_time_per_cycle_ms_serialised": t}
json.dump(res, open(out, "w"), indent=1)
print(json.dumps(res))
