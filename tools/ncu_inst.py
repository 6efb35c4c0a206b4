"""Executed warp-instructions per source line (per unit) from an ncu report.
usage: ncu_inst.py REP KERNEL_REGEX UNITS [MIN]"""
import csv, io, subprocess, sys
rep, kre, W = sys.argv[1], sys.argv[2], float(sys.argv[3])
mn = float(sys.argv[4]) if len(sys.argv) > 4 else 3
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--kernel-name", "regex:" + kre], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out))); cur = None; hdr = None; res = []
for r in rows:
    if len(r) >= 2 and r[0] == "File Path": cur = r[1].split("/")[-1]; continue
    if r and r[0] == "Line No": hdr = r; continue
    if hdr and r and r[0].isdigit():
        try: ie = int(r[hdr.index("Instructions Executed")])
        except ValueError: continue
        if ie: res.append((cur, int(r[0]), r[1].strip()[:80], ie))
tot = sum(x[3] for x in res); print("total per unit", round(tot / W, 1))
for f, l, s, ie in sorted(res, key=lambda x: (x[0], x[1])):
    if ie / W >= mn: print(f"{ie/W:7.1f} {f[:12]}:{l:<4d} {s}")
