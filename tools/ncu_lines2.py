"""Per-CUDA-source-line instruction counts / stall samples of one kernel in an ncu
report (cuda,sass view; inlined code is attributed to its innermost line).
usage: ncu_lines2.py REPORT KERNEL_SUBSTRING [TOP]"""
import csv, io, subprocess, sys
rep, ksub = sys.argv[1], sys.argv[2]
top = int(sys.argv[3]) if len(sys.argv) > 3 else 50
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                     capture_output=True, text=True).stdout
fpath = func = None
recs = []
for r in csv.reader(io.StringIO(out)):
    if not r: continue
    if r[0] == "File Path": fpath = r[1].split("/")[-1]; continue
    if r[0] == "Function Name": func = r[1]; continue
    if r[0] == "Line No" or r[0] == "": continue
    if ksub not in (func or ""): continue
    try:
        st, ex = int(r[4]), int(r[7])
    except (ValueError, IndexError):
        continue
    if ex or st:
        recs.append((fpath, int(r[0]), r[1].strip()[:72], ex, st))
tot = sum(x[3] for x in recs); tst = sum(x[4] for x in recs)
print(f"{ksub}: warp-instr {tot}, stall samples {tst}")
for x in sorted(recs, key=lambda x: -x[3])[:top]:
    print(f"{x[0][:16]:16s}{x[1]:5d} {100*x[3]/tot:5.1f}% {100*x[4]/max(tst,1):5.1f}%  {x[2]}")
