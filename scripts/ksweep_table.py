"""Table of an E_max sweep: python scripts/ksweep_table.py gpurun_out/ksweep/*.json"""
import json
import sys

print("| config | model | T | E_max | epoch ms | layer-edges/s | gather ms | gather GB/s | work items per layer / SPLIT rows per layer |")
print("|---|---|---|---|---|---|---|---|---|")
def key(p):
    parts = p.split("/")[-1][:-5].split("_")
    t = int(parts[2][1:]) if parts[2].startswith("T") else 128
    return (parts[:2], t, int(parts[-1]))


for f in sorted(sys.argv[1:], key=key):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception:
        continue
    c = d["config"]
    k = d["kernels"].get("gather_reduce") or d["kernels"].get("gat") or {}
    print(f"| {c['workload'].split(':')[0]} | {c['model']} | {key(f)[1]} | {c['E_max']} | {d['ms_per_step']:.2f} | {d['value']:.3g} | "
          f"{k.get('ms_per_step', 0):.2f} | {k.get('GB/s') or 0:.0f} | {'/'.join(str(q['items']) for q in c['plans'])} / {'/'.join(str(q['split_rows']) for q in c['plans'])} |")
