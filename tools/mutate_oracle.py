"""Mutation check of the oracle pins (CPU only).

Copies the repo to a scratch directory, applies one mutant at a time to
oracle/pfpl_oracle.c, rebuilds the oracle there and runs the oracle pin tests.
A mutant is KILLED when at least one test fails.  Usage:

    python tools/mutate_oracle.py            # all mutants
    python tools/mutate_oracle.py rel_scale  # one
"""
from __future__ import annotations

import os
import shutil
import subprocess
import sys
import tempfile

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))

# name -> (original text, mutated text, passage)
MUTANTS = {
    "rel_scale_f32": ("P->inv_w_f = 0.5f / lw;", "P->inv_w_f = 1.0f / lw;", "P:90 / R5"),
    "rel_scale_f64": ("P->inv_w_d = 0.5 / lw;", "P->inv_w_d = 1.0 / lw;", "P:90 / R5"),
    "noa_075": ("eps_abs = e > 0.0 ? nextafter(e, 0.0) : 0.0;",
                "eps_abs = e > 0.0 ? 0.75 * nextafter(e, 0.0) : 0.0;", "P:92 / R3"),
    "noa_no_rounddown": ("double r_lo = d > 0.0 ? nextafter(d, 0.0) : 0.0;",
                         "double r_lo = d > 0.0 ? nextafter(d, 1e300) : 0.0;", "P:92 / R3"),
    "tail_pad_zero": ("for (size_t i = m; i < cw; ++i) q[i] = q[m - 1];",
                      "for (size_t i = m; i < cw; ++i) q[i] = 0;", "R12"),
    "abs_inv_1": ("P->inv_f = 0.5f / ee;", "P->inv_f = 1.0f / ee;", "P:88"),
    "rel_no_shrink": ("float lo = flt_f(bits_f(a / P->c_lo_f) + 1u);",
                      "float lo = flt_f(bits_f(a / P->c_lo_f) + 0u);", "R7"),
    "rel_no_shrink_hi": ("float hi = flt_f(bits_f(a * P->c_lo_f) - 1u);",
                         "float hi = flt_f(bits_f(a * P->c_lo_f) - 0u);", "R7"),
    "rel64_no_shrink": ("double lo = flt_d(bits_d(a / P->c_lo_d) + 1u);",
                        "double lo = flt_d(bits_d(a / P->c_lo_d) + 0u);", "R7"),
    "abs_round_nearest": ("float ee = eps_abs > 0.0 ? round_down_f32(eps_abs) : 0.0f;",
                          "float ee = eps_abs > 0.0 ? (float)eps_abs : 0.0f;", "R1"),
    "repeat_pred_ff": ("    uint8_t prev = 0;\n    memset(M, 0, len / 8);",
                       "    uint8_t prev = 0xFF;\n    memset(M, 0, len / 8);", "R15"),
}

TESTS = ["tests/test_oracle_quant.py", "tests/test_oracle_stages.py",
         "tests/test_oracle_readings.py", "tests/test_boundcheck.py"]


def run(name: str) -> bool:
    orig, mut, cite = MUTANTS[name]
    with tempfile.TemporaryDirectory() as d:
        dst = os.path.join(d, "repo")
        shutil.copytree(ROOT, dst, ignore=shutil.ignore_patterns(
            ".git", "gpurun_out", "*.so", "__pycache__", ".hypothesis", "build*"))
        src = os.path.join(dst, "oracle", "pfpl_oracle.c")
        text = open(src).read()
        assert text.count(orig) == 1, f"{name}: pattern not found exactly once"
        open(src, "w").write(text.replace(orig, mut))
        r = subprocess.run([sys.executable, "-m", "pytest", "-q", "-x", "-m", "not gpu",
                            "-p", "no:randomly", *TESTS], cwd=dst, capture_output=True, text=True)
        killed = r.returncode != 0
        last = [ln for ln in r.stdout.splitlines() if ln.strip()][-1:] or [""]
        print(f"{name:18s} ({cite:9s}) {'KILLED' if killed else 'SURVIVED'}  {last[0]}")
        return killed


if __name__ == "__main__":
    names = sys.argv[1:] or list(MUTANTS)
    ok = all([run(n) for n in names])
    sys.exit(0 if ok else 1)
