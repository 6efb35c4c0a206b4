"""Summarise an ncu report: key SOL metrics, stall reasons, per-opcode mix, top stall PCs."""
import csv, subprocess, sys, io
from collections import Counter
rep = sys.argv[1]
def raw():
    out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv"], capture_output=True, text=True).stdout
    r = list(csv.reader(io.StringIO(out)))
    return r
r = raw()
hdr, units = r[0], r[1]
for vals in r[2:]:
    d = dict(zip(hdr, vals))
    print("kernel:", d.get("Kernel Name", "")[:90])
    keys = ["gpu__time_duration.sum", "sm__throughput.avg.pct_of_peak_sustained_elapsed",
            "dram__bytes_read.sum", "dram__bytes_write.sum", "gpu__dram_throughput.avg.pct_of_peak_sustained_elapsed",
            "smsp__inst_executed.sum", "sm__warps_active.avg.pct_of_peak_sustained_active",
            "launch__registers_per_thread", "launch__occupancy_limit_registers", "launch__occupancy_limit_shared_mem",
            "smsp__issue_active.avg.pct_of_peak_sustained_active",
            "sm__inst_executed_pipe_alu.avg.pct_of_peak_sustained_active",
            "sm__inst_executed_pipe_fma.avg.pct_of_peak_sustained_active",
            "sm__inst_executed_pipe_lsu.avg.pct_of_peak_sustained_active",
            "sm__inst_executed_pipe_xu.avg.pct_of_peak_sustained_active",
            "l1tex__data_bank_conflicts_pipe_lsu_mem_shared.sum",
            "l1tex__data_pipe_lsu_wavefronts_mem_shared.sum"]
    for k in keys:
        if k in d:
            print(f"  {k:60s} {d[k]:>16s} {units[hdr.index(k)]}")
    st = [(k, float(v.replace(',', ''))) for k, v in d.items()
          if k.startswith("smsp__pcsamp_warps_issue_stalled_") and not k.endswith("not_issued") and v]
    tot = sum(v for _, v in st)
    for k, v in sorted(st, key=lambda x: -x[1])[:10]:
        print(f"  stall {k[33:]:40s} {100*v/tot:5.1f}%")
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "sass"],
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
h = rows[1]; data = rows[2:]
ia, isrc, ist, iex = h.index("Address"), h.index("Source"), h.index("Warp Stall Sampling (All Samples)"), h.index("Instructions Executed")
c, s = Counter(), Counter(); tot = 0; recs = []
for x in data:
    try: ex = int(x[iex] or 0); stl = int(x[ist] or 0)
    except Exception: continue
    op = x[isrc].split()[0] if x[isrc] else "?"
    if op.startswith("@"): op = x[isrc].split()[1]
    op = op.split(".")[0]
    c[op] += ex; s[op] += stl; tot += ex; recs.append((x[ia], x[isrc], ex, stl))
print("executed warp-instr:", tot)
for op, n in c.most_common(int(sys.argv[2]) if len(sys.argv) > 2 else 18):
    print(f"  {op:10s} {n:11d} {100*n/tot:5.1f}%  stall-samples {s[op]}")
print("top stall PCs:")
for a, src, ex, stl in sorted(recs, key=lambda x: -x[3])[:12]:
    print("  ", a[-5:], src[:64].ljust(64), ex, stl)
