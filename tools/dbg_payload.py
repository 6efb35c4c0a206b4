import sys; sys.path.insert(0,'.')
import numpy as np, torch, synth, oracle
import paper_conf_ipps_fallinadcb25_b200 as pk
for dt, n in ((np.float64, 31), (np.float64, 2048), (np.float32, 31)):
    spec = synth.FieldSpec("t", (n,), "f32" if dt == np.float32 else "f64", 3, A=0.5, tau=0.01)
    x = synth.generate(spec).numpy()
    g = pk.compress(torch.from_numpy(x).cuda(), "abs", 1e-2).cpu().numpy().tobytes()
    c = oracle.compress(x, "abs", 1e-2)
    print(dt.__name__, n, len(g), len(c), g == c)
    print(" gpu", g[48:].hex())
    print(" cpu", c[48:].hex())
