#!/usr/bin/env python
"""Per-CUDA-source-line instruction and stall-sample shares of an ncu report
(needs -lineinfo and --import-source on):  ncu_lines.py <report> [top]"""
import csv, io, subprocess, sys
rep = sys.argv[1]
top = int(sys.argv[2]) if len(sys.argv) > 2 else 50
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
fname, agg = "?", {}
for r in rows:
    if len(r) == 2 and r[0] == "File Path":
        fname = r[1].split("/")[-1]
        continue
    if len(r) < 8 or not r[0].isdigit():
        continue
    try:
        s, e = float(r[4] or 0), float(r[7] or 0)
    except ValueError:
        continue
    if s or e:
        agg[(fname, int(r[0]))] = (s, e, r[1].strip()[:90])
tS = sum(v[0] for v in agg.values()) or 1
tE = sum(v[1] for v in agg.values()) or 1
print(f"stall samples {tS:.0f}, warp instructions executed {tE:.4g}")
for k, (s, e, src) in sorted(agg.items(), key=lambda x: -x[1][0])[:top]:
    print(f"{k[0][:14]:14s}:{k[1]:<5d} stall {100 * s / tS:5.1f}%  instr {100 * e / tE:5.1f}%  {src}")
