"""Per-stage SASS instruction budget of the fused encoder/decoder from an ncu
report (`--set full --import-source on`): executed warp-instructions per CUDA
source line (inlined code attributed to its innermost line), grouped into the
pipeline stages of DESIGN.md 7.1 and expressed as thread-instructions per
element (warp-instr * 32 / n).

usage: python tools/ncu_budget.py REPORT KERNEL_SUBSTRING N_ELEMENTS [--lines]
"""
import csv
import io
import subprocess
import sys
from collections import defaultdict

# device.cuh helpers are attributed by the "// [stage]" section markers of the
# sources (see stage_map), i.e. by what they implement
STAGES = []


def stage_map():
    """(file, first line, last line, stage) from the "// [stage] NAME" markers."""
    import os
    import re
    root = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
    extra = []
    for fn in ("pfpl_encode.cuh", "pfpl_decode.cuh", "pfpl_device.cuh"):
        lines = open(os.path.join(root, "paper_conf_ipps_fallinadcb25_b200", "csrc", fn)).read().splitlines()
        marks = [(i + 1, m.group(1)) for i, l in enumerate(lines) if (m := re.search(r"// \[stage\] (.+)$", l))]
        for j, (ln, name) in enumerate(marks):
            end = marks[j + 1][0] - 1 if j + 1 < len(marks) else len(lines)
            extra.append((fn, ln, end, name))
    return extra


def load(rep, ksub):
    out = subprocess.run(["ncu", "-i", rep, "--page", "source", "--csv", "--print-source", "cuda,sass"],
                         capture_output=True, text=True).stdout
    fpath = func = None
    recs = defaultdict(lambda: [0, 0, ""])
    for r in csv.reader(io.StringIO(out)):
        if not r:
            continue
        if r[0] == "File Path":
            fpath = r[1].split("/")[-1]
            continue
        if r[0] == "Function Name":
            func = r[1]
            continue
        if r[0] in ("Line No", ""):
            continue
        if ksub not in (func or ""):
            continue
        try:
            st, ex = int(r[4]), int(r[7])
        except (ValueError, IndexError):
            continue
        k = (fpath, int(r[0]))
        recs[k][0] += ex
        recs[k][1] += st
        recs[k][2] = r[1].strip()[:80]
    return recs


def stage_of(f, ln, extra):
    for ff, a, b, name in extra + STAGES:
        if f.startswith(ff) and a <= ln <= b:
            return name
    return f"other ({f})"


def main():
    rep, ksub, n = sys.argv[1], sys.argv[2], float(sys.argv[3])
    extra = stage_map()
    recs = load(rep, ksub)
    tot = sum(v[0] for v in recs.values())
    tst = sum(v[1] for v in recs.values()) or 1
    agg = defaultdict(lambda: [0, 0])
    for (f, ln), (ex, st, _) in recs.items():
        s = stage_of(f, ln, extra)
        agg[s][0] += ex
        agg[s][1] += st
    print(f"{ksub}: {tot} warp-instructions = {tot * 32 / n:.2f} thread-instructions per element (n = {n:.0f})")
    print(f"{'stage':45s} {'instr/elem':>10s} {'share':>7s} {'stalls':>7s}")
    for s, (ex, st) in sorted(agg.items(), key=lambda kv: -kv[1][0]):
        print(f"{s[:45]:45s} {ex * 32 / n:10.2f} {100 * ex / tot:6.1f}% {100 * st / tst:6.1f}%")
    if "--lines" in sys.argv:
        for (f, ln), (ex, st, src) in sorted(recs.items(), key=lambda kv: -kv[1][0])[:60]:
            print(f"{f[:16]:16s}{ln:5d} {stage_of(f, ln, extra)[:20]:20s} {ex * 32 / n:6.2f} {src}")


if __name__ == "__main__":
    main()
