"""Per-source-line stall samples (by reason) and executed warp-instructions from an ncu report.
usage: ncu_stalls.py REP KERNEL_REGEX [TOP]"""
import csv, io, subprocess, sys
from collections import Counter
rep, kre = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass",
                      "--kernel-name", "regex:" + kre], capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
cur = None; hdr = None; res = []
for r in rows:
    if len(r) >= 2 and r[0] == "File Path": cur = r[1].split("/")[-1]; continue
    if r and r[0] == "Line No": hdr = r; continue
    if hdr and r and r[0].isdigit():
        st = Counter()
        for i, k in enumerate(hdr):
            if k.startswith("stall_") and "Not Issued" not in k and i < len(r):
                try: st[k[6:]] += int(r[i])
                except ValueError: pass
        try: ie = int(r[hdr.index("Instructions Executed")])
        except ValueError: ie = 0
        res.append(((cur, int(r[0])), r[1].strip()[:58], st, ie))
tot = Counter()
for _, _, c, _ in res: tot.update(c)
T = sum(tot.values()) or 1
print("total samples", T, {k: f"{100*v/T:.1f}%" for k, v in tot.most_common(9)})
for ln, s, c, ie in sorted(res, key=lambda x: -sum(x[2].values()))[:top]:
    n = sum(c.values())
    print(f"{100*n/T:5.1f}% {ie/1e6:7.2f}M {ln[0][:14]}:{ln[1]:<4d} {s:58s} " +
          " ".join(f"{k}:{100*v/T:.1f}" for k, v in c.most_common(3)))
