"""Summarise an `ncu --set full` report of bench.py into profiles/ (per-kernel table + the
per-launch DRAM traffic bench.py reports as roofline.traffic).

usage: python scripts/ncu_summary.py REPORT.ncu-rep CONFIG OUT_SUMMARY.json [TRAFFIC.json]
Kernel launches are grouped like bench.py's per-kernel events: when fast / distribute run as
two launches per extract (SS_FAST_SPLIT=1, round 1), the smaller grid of the pair is level 0's.
"""
import csv
import io
import json
import subprocess
import sys

METRICS = ["gpu__time_duration.sum", "dram__bytes_read.sum", "dram__bytes_write.sum", "launch__grid_size",
           "launch__block_size", "launch__registers_per_thread", "smsp__inst_executed.sum",
           "sm__warps_active.avg.pct_of_peak_sustained_active", "sm__inst_executed.avg.per_cycle_active",
           "lts__t_sectors.sum"]
SHORT = {"fast_bands_kernel": "fast", "distribute_kernel": "distribute", "pyramid_fused_kernel": "pyramid",
         "describe_kernel": "describe", "match_prepare": "match_prepare", "match_window_kernel": "match_window",
         "match_window_resolve": "match_resolve", "brute_tc_kernel": "brute_tc", "brute_expand_kernel": "brute_expand",
         "match_brute_merge": "brute_merge", "lastframe_kernel": "lastframe", "project_kernel": "project",
         "brute_shard_top2": "brute_shard_top2", "brute_parts_merge": "brute_parts_merge",
         "stereo_match_kernel": "stereo", "stereo_outlier_kernel": "stereo_outliers",
         "distribute_grid_kernel": "distribute_grid"}


def main():
    rep, cfg, out = sys.argv[1], sys.argv[2], sys.argv[3]
    traffic_path = sys.argv[4] if len(sys.argv) > 4 else None
    txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics", ",".join(METRICS)],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(txt)))
    hdr, units = rows[0], rows[1]
    launches = []
    for r in rows[2:]:
        d = dict(zip(hdr, r))
        full = d["Kernel Name"]
        hits = [k for k in SHORT if k in full]  # template instances, e.g. describe_kernel<(bool)0>
        name = max(hits, key=len) if hits else full.split("(")[0].split("::")[-1]
        rec = {"kernel": SHORT.get(name, name)}
        for m in METRICS:
            u = units[hdr.index(m)]
            v = float(d[m].replace(",", "")) if d[m] else None
            if v is not None and u in ("Kbyte", "Mbyte", "Gbyte"):
                v *= {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}[u]
            if v is not None and u == "ns":
                v /= 1e3
            if v is not None and u == "ms":
                v *= 1e3
            rec[m] = v
        launches.append(rec)
    # level-0 vs levels >= 1 by grid size within each kind
    for kind in ("fast", "distribute"):
        grids = sorted({x["launch__grid_size"] for x in launches if x["kernel"] == kind})
        if len(grids) < 2:  # one launch per extract (the default since round 2): keep the name
            continue
        for x in launches:
            if x["kernel"] == kind:
                x["kernel"] = f"{kind}_l0" if x["launch__grid_size"] == grids[0] else f"{kind}_l1plus"
    summary = {}
    for x in launches:
        s = summary.setdefault(x["kernel"], {"launches": 0})
        s["launches"] += 1
        for m in METRICS:
            if x[m] is not None:
                s[m] = s.get(m, 0.0) + x[m]
    for k, s in summary.items():
        n = s.pop("launches")
        for m in METRICS:
            if m in s:
                s[m] = round(s[m] / n, 3)
        s["launches_captured"] = n
        s["dram_bytes_per_launch"] = round(s.get("dram__bytes_read.sum", 0) + s.get("dram__bytes_write.sum", 0))
    doc = {"report": rep.split("/")[-1], "config": cfg,
           "note": "ncu --set full --clock-control none (cache flushed between kernels by ncu: cold-cache DRAM "
                   "bytes, serialised launches); per-launch averages; times in us, bytes in bytes",
           "kernels": summary}
    with open(out, "w") as f:
        json.dump(doc, f, indent=1)
    if traffic_path:
        try:
            with open(traffic_path) as f:
                tr = json.load(f)
        except FileNotFoundError:
            tr = {}
        tr[cfg] = {k: s["dram_bytes_per_launch"] for k, s in summary.items()}
        tr["_note"] = "dram__bytes_read.sum + dram__bytes_write.sum per launch from ncu --set full (cold cache)"
        with open(traffic_path, "w") as f:
            json.dump(tr, f, indent=1, sort_keys=True)
    for k, s in sorted(summary.items()):
        print(f"{k:18s} {s['gpu__time_duration.sum']:8.2f} us  dram {s['dram_bytes_per_launch'] / 1e6:7.3f} MB  "
              f"inst {s['smsp__inst_executed.sum'] / 1e6:6.2f} M  ipc {s.get('sm__inst_executed.avg.per_cycle_active', 0):.2f}")


if __name__ == "__main__":
    main()
