"""Executed-instruction mix (by SASS opcode) of one kernel launch from an ncu report with
source import.  Usage: python scripts/ncu_sass_mix.py REPORT KERNEL_REGEX [launch_index] [top]"""
import csv
import io
import subprocess
import sys

rep, krx = sys.argv[1], sys.argv[2]
li = int(sys.argv[3]) if len(sys.argv) > 3 else 0
top = int(sys.argv[4]) if len(sys.argv) > 4 else 30
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass", "-k", f"regex:{krx}",
                      "--launch-skip", str(li), "--launch-count", "1"], capture_output=True, text=True).stdout
mix, h = {}, None
for r in csv.reader(io.StringIO(out)):
    if r and r[0] == "Address":
        h = {n: i for i, n in enumerate(r)}
        continue
    if not h or not r or not r[0].startswith("0x"):
        continue
    ins = r[h["Source"]].strip()
    if ins.startswith("@"):
        ins = ins.split(None, 1)[1]
    op = ins.split()[0] if ins else "?"
    try:
        n = float(r[h["Instructions Executed"]] or 0)
    except ValueError:
        continue
    mix[op] = mix.get(op, 0.0) + n
tot = sum(mix.values()) or 1
print(f"total warp instructions {tot:.0f}")
for op, n in sorted(mix.items(), key=lambda x: -x[1])[:top]:
    print(f"{op:24s} {n:12.0f} {100 * n / tot:5.1f}%")
