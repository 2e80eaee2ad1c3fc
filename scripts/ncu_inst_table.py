"""Per-kernel executed warp instructions, device time and pipe utilisation per tick from an
ncu --metrics CSV (scripts/gpu_inst.sh).  Usage: python scripts/ncu_inst_table.py CSV [ticks]"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
ticks = float(sys.argv[2]) if len(sys.argv) > 2 else None
hdr = None
launch = {}
for r in rows:
    if r and r[0] == "ID":
        hdr = {n: i for i, n in enumerate(r)}
        continue
    if not hdr or len(r) < len(hdr):
        continue
    lid = r[hdr["ID"]]
    name = r[hdr["Kernel Name"]].split("(")[0].replace("(anonymous namespace)::", "").split("::")[-1]
    d = launch.setdefault(lid, {"name": name})
    try:
        d[r[hdr["Metric Name"]]] = float(r[hdr["Metric Value"]].replace(",", ""))
    except ValueError:
        d[r[hdr["Metric Name"]]] = r[hdr["Metric Value"]]
agg = {}
for d in launch.values():
    a = agg.setdefault(d["name"], {"n": 0, "inst": 0.0, "us": 0.0, "alu": 0.0, "fma": 0.0, "lsu": 0.0, "xu": 0.0, "warps": 0.0})
    a["n"] += 1
    a["inst"] += d.get("smsp__inst_executed.sum", 0)
    a["us"] += d.get("gpu__time_duration.sum", 0) / 1000.0
    for k, m in (("alu", "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active"),
                 ("fma", "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active"),
                 ("lsu", "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active"),
                 ("xu", "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active"),
                 ("warps", "sm__warps_active.avg.pct_of_peak_sustained_active")):
        a[k] += d.get(m, 0)
tot = sum(a["inst"] for a in agg.values())
T = ticks or max(a["n"] for a in agg.values())
print(f"{'kernel':24s} {'launches':>8s} {'Minst/tick':>10s} {'share':>6s} {'us/launch':>9s} {'alu%':>5s} {'fma%':>5s} {'lsu%':>5s} {'xu%':>5s} {'warps%':>6s}")
for n, a in sorted(agg.items(), key=lambda x: -x[1]["inst"]):
    k = a["n"]
    print(f"{n:24s} {k:8d} {a['inst'] / T / 1e6:10.3f} {a['inst'] / tot:6.1%} {a['us'] / k:9.2f} {a['alu'] / k:5.1f} {a['fma'] / k:5.1f} "
          f"{a['lsu'] / k:5.1f} {a['xu'] / k:5.1f} {a['warps'] / k:6.1f}")
print(f"total {tot / T / 1e6:.2f} M warp instructions per tick ({T:g} ticks)")
