"""Ordered per-launch list of the last N launches of an ncu launch CSV:
python scripts/launch_seq.py file.csv N"""
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, data = None, []
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d["Metric Name"] == "gpu__time_duration.sum":
            v = float(d["Metric Value"])
            u = d["Metric Unit"]
            v = v / 1e6 if u == "ns" else (v / 1e3 if u in ("us", "usecond") else v)
            data.append((d["Kernel Name"][:90], d.get("Grid Size", ""), v))
n = int(sys.argv[2]) if len(sys.argv) > 2 else 60
tot = 0.0
for k, g, v in data[-n:]:
    tot += v
    print(f"{v:8.3f} ms  {g:>16s}  {k}")
print(f"total {tot:.2f} ms over {min(n, len(data))} launches")
