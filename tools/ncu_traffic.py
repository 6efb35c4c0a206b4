"""Merge per-launch DRAM traffic (dram__bytes_read.sum + dram__bytes_write.sum) of
the encoder/decoder from an `ncu --set full` report into profiles/traffic.json,
which bench.py reports as roofline.traffic.
usage: ncu_traffic.py REP CONFIG/BOUND [SOURCE-NOTE]"""
import csv, io, json, os, subprocess, sys
rep, key = sys.argv[1], sys.argv[2]
note = sys.argv[3] if len(sys.argv) > 3 else rep
out = subprocess.run(["ncu", "-i", rep, "--page", "raw", "--csv", "--metrics",
                      "dram__bytes_read.sum,dram__bytes_write.sum"], capture_output=True, text=True).stdout
r = list(csv.reader(io.StringIO(out)))
hdr, units = r[0], r[1]
scale = {"byte": 1, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9}
f = os.path.join(os.path.dirname(os.path.dirname(os.path.abspath(__file__))), "profiles", "traffic.json")
t = json.load(open(f)) if os.path.exists(f) else {}
ent = t.get(key, {})
for vals in r[2:]:
    d = dict(zip(hdr, vals)); u = dict(zip(hdr, units))
    name = d["Kernel Name"]
    kind = "encode" if "encode_kernel" in name else "decode" if "decode_kernel" in name else None
    if not kind:
        continue
    b = sum(float(d[m].replace(",", "")) * scale[u[m]] for m in ("dram__bytes_read.sum", "dram__bytes_write.sum"))
    ent[kind] = int(b)
    print(key, kind, name[:60], int(b))
t[key] = ent
t["source"] = note
json.dump(t, open(f, "w"), indent=1)
