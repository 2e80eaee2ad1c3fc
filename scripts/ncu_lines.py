"""Aggregate an ncu report's per-SASS metrics by CUDA source line.

usage: python scripts/ncu_lines.py REPORT.ncu-rep KERNEL_REGEX [top_n]
Needs a report captured with --import-source on from a -lineinfo build.
"""
import csv
import io
import subprocess
import sys


def main():
    rep, kern = sys.argv[1], sys.argv[2]
    top = int(sys.argv[3]) if len(sys.argv) > 3 else 25
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                          "--kernel-name", f"regex:{kern}", "--launch-count", "1"],
                         capture_output=True, text=True).stdout
    rows = list(csv.reader(io.StringIO(out)))
    hdr = None
    agg = {}
    cur_file, cur_line, cur_src = "", None, ""
    for r in rows:
        if not r:
            continue
        if r[0] == "File Path":
            cur_file = r[1].split("/")[-1]
            continue
        if r[0] == "Line No":
            hdr = r
            continue
        if hdr is None:
            continue
        if r[0] not in ("",):
            cur_line, cur_src = r[0], r[1]
            continue
        if len(r) < len(hdr) or r[2] in ("-", "..."):
            continue
        try:
            ex = float(r[hdr.index("Instructions Executed")] or 0)
            st = float(r[hdr.index("Warp Stall Sampling (All Samples)")] or 0)
        except ValueError:
            continue
        key = (cur_file, cur_line)
        a = agg.setdefault(key, [0.0, 0.0, cur_src])
        a[0] += ex
        a[1] += st
    tot_e = sum(v[0] for v in agg.values()) or 1
    tot_s = sum(v[1] for v in agg.values()) or 1
    print(f"total warp instructions {tot_e:.0f}, stall samples {tot_s:.0f}")
    for (f, ln), (e, s, src) in sorted(agg.items(), key=lambda kv: -kv[1][1])[:top]:
        print(f"{f}:{ln:>5s} instr {100 * e / tot_e:5.1f}%  stall {100 * s / tot_s:5.1f}%  {src.strip()[:90]}")


if __name__ == "__main__":
    main()
