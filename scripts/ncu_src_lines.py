"""Per-CUDA-source-line instruction counts and stall samples of one kernel launch from an
ncu report captured with --import-source on (scripts/gpu_ncu_src.sh).
Usage: python scripts/ncu_src_lines.py REPORT KERNEL_REGEX [launch_index] [top]"""
import csv
import io
import subprocess
import sys

rep, krx = sys.argv[1], sys.argv[2]
li = int(sys.argv[3]) if len(sys.argv) > 3 else 0
top = int(sys.argv[4]) if len(sys.argv) > 4 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass", "-k", f"regex:{krx}",
                      "--launch-skip", str(li), "--launch-count", "1"], capture_output=True, text=True).stdout
data, h, fname = [], None, ""
for r in csv.reader(io.StringIO(out)):
    if r and r[0] == "File Path":
        fname = r[1].rsplit("/", 1)[-1]
    elif r and r[0] == "Line No":
        h = {n: i for i, n in enumerate(r) if n not in ("Source",)}
        h["Source"] = 1
    elif h and r and r[0] not in ("", "Function Name"):
        try:
            inst = float(r[h["Instructions Executed"]] or 0)
            samp = float(r[h["Warp Stall Sampling (All Samples)"]] or 0)
        except (ValueError, IndexError):
            continue
        if inst or samp:
            data.append((inst, samp, f"{fname}:{r[0]}", r[1].strip()[:100]))
tot_i = sum(d[0] for d in data) or 1
tot_s = sum(d[1] for d in data) or 1
print(f"total warp instructions {tot_i:.0f}, stall samples {tot_s:.0f}")
for inst, samp, line, src in sorted(data, key=lambda d: -d[0])[:top]:
    print(f"{100 * inst / tot_i:5.1f}% inst {100 * samp / tot_s:5.1f}% samp  {line:>18} {src}")
