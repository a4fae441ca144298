"""Per-kernel totals of an ncu launch list: python scripts/launch_table.py file.csv [n]"""
import collections
import csv
import sys

rows = list(csv.reader(open(sys.argv[1])))
hdr, data = None, []
for r in rows:
    if r and r[0] == "ID":
        hdr = r
        continue
    if hdr and len(r) == len(hdr):
        data.append(dict(zip(hdr, r)))
agg = collections.defaultdict(lambda: [0, 0.0])
for d in data:
    if d["Metric Name"] != "gpu__time_duration.sum":
        continue
    v = float(d["Metric Value"])
    v = v / 1e6 if d["Metric Unit"] == "ns" else (v / 1e3 if d["Metric Unit"] in ("us", "usecond") else v)
    k = d["Kernel Name"][:100]
    agg[k][0] += 1
    agg[k][1] += v
tot = sum(v[1] for v in agg.values())
print(f"{sys.argv[1]}: total {tot:.2f} ms over {sum(v[0] for v in agg.values())} launches")
for k, v in sorted(agg.items(), key=lambda x: -x[1][1])[: int(sys.argv[2]) if len(sys.argv) > 2 else 20]:
    print(f"  {v[1]:9.3f} ms x{v[0]:4d}  {k}")
