"""Per-source-line executed instruction counts and opcode mix from an ncu report."""
import csv, io, subprocess, sys
from collections import defaultdict, Counter
rep = sys.argv[1]; per = float(sys.argv[2]) if len(sys.argv) > 2 else 1.0
top = int(sys.argv[3]) if len(sys.argv) > 3 else 40
out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"] + (["--kernel-name", "regex:" + sys.argv[4]] if len(sys.argv) > 4 else []),
                     capture_output=True, text=True).stdout
rows = list(csv.reader(io.StringIO(out)))
cur = None; line = None; agg = defaultdict(Counter); src = {}
ALU = {"LOP3", "SHF", "ISETP", "IADD3", "SEL", "FSETP", "PRMT", "LEA", "VIADD", "FMNMX", "PLOP3", "POPC", "FLO", "BMSK", "ISCADD", "P2R", "R2P", "VIMNMX"}
for r in rows:
    if len(r) >= 2 and r[0] == "File Path": cur = r[1].split("/")[-1]; continue
    if len(r) > 8 and r[0].isdigit() and r[2] == "-":
        line = (cur, int(r[0])); src[line] = r[1].strip()[:70]; continue
    if len(r) > 8 and r[0] == "" and r[2] != "-" and line:
        s = r[3]; ex = r[7]
        try: ex = int(ex)
        except: continue
        op = s.split()[0] if s else "?"
        if op.startswith("@"): op = s.split()[1]
        op = op.split(".")[0]
        agg[line][op] += ex
tot = sum(sum(c.values()) for c in agg.values())
alu = lambda c: sum(v for k, v in c.items() if k in ALU)
print(f"total {tot}  ALU {sum(alu(c) for c in agg.values())}")
for ln, c in sorted(agg.items(), key=lambda kv: -alu(kv[1]))[:top]:
    n = sum(c.values())
    print(f"{alu(c)/per:8.1f} alu {n/per:8.1f} all  {ln[0]}:{ln[1]:<4d} {src.get(ln,'')[:60]:60s} {dict(c.most_common(4))}")
