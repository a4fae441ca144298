"""Per-launch DRAM traffic of a kernel class from an `ncu --set full` raw CSV
(`ncu -i rep --page raw --csv`) covering one step's launches of that class;
merges it into profiles/ncu_traffic.json, which bench.py reports as
roofline.traffic (dram__bytes_read.sum + dram__bytes_write.sum per launch).

    python scripts/ncu_traffic.py <raw.csv> <config:model:class> <kernel regex> [source note]
"""
import csv
import json
import os
import re
import sys

ROOT = os.path.dirname(os.path.dirname(os.path.abspath(__file__)))
UNIT = {"byte": 1.0, "Kbyte": 1e3, "Mbyte": 1e6, "Gbyte": 1e9, "Tbyte": 1e12}


def main(path, key, regex, note=""):
    rows = list(csv.reader(open(path)))
    h, u = rows[0], rows[1]
    ik = h.index("Kernel Name")
    ir, iw = h.index("dram__bytes_read.sum"), h.index("dram__bytes_write.sum")
    it = h.index("gpu__time_duration.sum")
    vals, times = [], []
    for r in rows[2:]:
        if not re.search(regex, r[ik]):
            continue
        vals.append(float(r[ir]) * UNIT[u[ir]] + float(r[iw]) * UNIT[u[iw]])
        times.append(float(r[it]))
    if not vals:
        raise SystemExit(f"no launch of {regex} in {path}")
    out = os.path.join(ROOT, "profiles", "ncu_traffic.json")
    d = json.load(open(out)) if os.path.exists(out) else {}
    d[key] = {"bytes_per_launch": sum(vals) / len(vals), "launches": len(vals),
              "per_launch_bytes": vals, "per_launch_time": times, "time_unit": u[it],
              "source": os.path.basename(path) + (f" ({note})" if note else "")}
    json.dump(d, open(out, "w"), indent=1)
    print(key, d[key]["bytes_per_launch"] / 1e9, "GB per launch over", len(vals), "launches")


if __name__ == "__main__":
    main(*sys.argv[1:])
