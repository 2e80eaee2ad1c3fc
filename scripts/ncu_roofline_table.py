"""Per-kernel roofline table from `ncu --set full` reports (the north_star's ask: achieved HBM
GB/s against the B200 peak for the pyramid, FAST and descriptor kernels; integer / tensor pipe
utilisation for the matchers).

usage: python scripts/ncu_roofline_table.py OUT.json REPORT.ncu-rep [REPORT2.ncu-rep ...]
Peaks: MEASURED_PEAKS.json hbm_gbs when present (else the B200_PROFILING.md fallback)."""
import csv
import re
import io
import json
import os
import subprocess
import sys

M = {"t_us": "gpu__time_duration.sum", "dram_rd": "dram__bytes_read.sum", "dram_wr": "dram__bytes_write.sum",
     "dram_pct": "dram__throughput.avg.pct_of_peak_sustained_elapsed",
     "alu_pct": "sm__pipe_alu_cycles_active.avg.pct_of_peak_sustained_active",
     "fma_pct": "sm__pipe_fma_cycles_active.avg.pct_of_peak_sustained_active",
     "tensor_pct": "TPC.TriageCompute.sm__pipe_tensor_cycles_active_realtime.avg.pct_of_peak_sustained_elapsed",
     "lsu_pct": "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
     "l2_hit_pct": "lts__t_sector_hit_rate.pct", "ipc": "sm__inst_executed.avg.per_cycle_active",
     "warps_active_pct": "sm__warps_active.avg.pct_of_peak_sustained_active", "grid": "launch__grid_size",
     "block": "launch__block_size"}
SCALE = {"Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "byte": 1.0, "ns": 1e-3, "us": 1.0, "usecond": 1.0,
         "nsecond": 1e-3, "msecond": 1e3, "ms": 1e3}


def peaks():
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    try:
        d = json.load(open(os.path.join(root, "MEASURED_PEAKS.json")))
        return float(d["hbm_gbs"]), "MEASURED_PEAKS.json"
    except Exception:
        return 6650.0, "B200_PROFILING.md fallback"


def main():
    out, reps = sys.argv[1], sys.argv[2:]
    hbm, src = peaks()
    rows = {}
    for rep in reps:
        txt = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics", ",".join(M.values())],
                             capture_output=True, text=True).stdout
        r = list(csv.reader(io.StringIO(txt)))
        hdr, units = r[0], r[1]
        for row in r[2:]:
            d = dict(zip(hdr, row))
            full = d["Kernel Name"].replace("(anonymous namespace)", "anon").replace("<unnamed>", "anon")
            while re.search(r"<[^<>]*>", full):  # template arguments, e.g. describe_kernel<(bool)0>
                full = re.sub(r"<[^<>]*>", "", full)
            name = full.split("(")[0].split("::")[-1]
            rec = {}
            for k, m in M.items():
                if m not in d or d[m] in ("", "n/a", "no data"):
                    continue
                v = float(d[m].replace(",", ""))
                v *= SCALE.get(units[hdr.index(m)], 1.0)
                rec[k] = v
            rows.setdefault(name, []).append(rec)
    table = {}
    for name, recs in rows.items():
        avg = {k: sum(x.get(k, 0.0) for x in recs) / len(recs) for k in recs[0]}
        gbs = (avg.get("dram_rd", 0) + avg.get("dram_wr", 0)) / (avg["t_us"] * 1e-6) / 1e9
        table[name] = {"launches": len(recs), "time_us": round(avg["t_us"], 2),
                       "dram_bytes": round(avg.get("dram_rd", 0) + avg.get("dram_wr", 0)),
                       "achieved_dram_gbs": round(gbs, 1), "pct_of_hbm_peak": round(100 * gbs / hbm, 2),
                       **{k: round(avg[k], 2) for k in ("dram_pct", "alu_pct", "fma_pct", "tensor_pct", "lsu_pct",
                                                         "l2_hit_pct", "ipc", "warps_active_pct") if k in avg},
                       "grid": int(avg.get("grid", 0)), "block": int(avg.get("block", 0))}
    doc = {"reports": [os.path.basename(x) for x in reps], "hbm_peak_gbs": hbm, "peak_src": src,
           "note": "ncu --set full --clock-control none: each launch replayed with cold caches and serialised, so "
                   "DRAM bytes are cold-cache and times are per launch alone; pct_of_hbm_peak = (DRAM read + write) "
                   "/ time vs the measured copy bandwidth; alu / fma / tensor = pipe utilisation while active",
           "kernels": table}
    json.dump(doc, open(out, "w"), indent=1)
    for k, v in sorted(table.items(), key=lambda kv: -kv[1]["time_us"]):
        print(f"{k:28s} {v['time_us']:8.1f} us  {v['achieved_dram_gbs']:8.1f} GB/s ({v['pct_of_hbm_peak']:5.1f}% HBM)  "
              f"alu {v.get('alu_pct', 0):5.1f}%  tensor {v.get('tensor_pct', 0):5.1f}%  ipc {v.get('ipc', 0):.2f}")


if __name__ == "__main__":
    main()
