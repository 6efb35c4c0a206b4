"""Run individual compress/decompress cases in subprocesses with a timeout."""
import subprocess, sys, itertools
CASE = r'''
import sys, numpy as np, torch
sys.path.insert(0, ".")
import paper_conf_ipps_fallinadcb25_b200 as pk
dt, bound, kind, n = sys.argv[1], sys.argv[2], sys.argv[3], int(sys.argv[4])
npdt = np.float32 if dt == "f32" else np.float64
rng = np.random.default_rng(7)
if kind == "rand":
    u = rng.integers(0, 2**63, size=n, dtype=np.int64).astype(np.uint64)
    x = (u.astype(np.uint32) if npdt == np.float32 else u).view(npdt)
elif kind == "const":
    x = np.full(n, 2.5, npdt)
else:
    x = np.zeros(n, npdt)
xd = torch.from_numpy(x).cuda()
s = pk.compress(xd, bound, 1e-3)
torch.cuda.synchronize()
y = pk.decompress(s)
torch.cuda.synchronize()
print("ok", len(s))
'''
open("/tmp/case.py", "w").write(CASE)
for dt, bound, kind, n in itertools.product(["f64", "f32"], ["abs", "rel", "noa"], ["rand", "const", "zero"], [5 * 2048 + 3, 3 * 4096]):
    try:
        r = subprocess.run([sys.executable, "/tmp/case.py", dt, bound, kind, str(n)], capture_output=True, text=True, timeout=40)
        print(dt, bound, kind, n, r.stdout.strip()[-40:], r.stderr.strip()[-200:], flush=True)
    except subprocess.TimeoutExpired:
        print(dt, bound, kind, n, "HANG", flush=True)
