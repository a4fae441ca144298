"""Table of an E_max sweep: python scripts/ksweep_table.py gpurun_out/ksweep/*.json"""
import json
import sys

print("| config | model | E_max | epoch ms | layer-edges/s | gather ms | gather GB/s | work items per layer / SPLIT rows per layer |")
print("|---|---|---|---|---|---|---|---|")
for f in sorted(sys.argv[1:], key=lambda p: (p.split("/")[-1].split("_")[:2], int(p.split("_")[-1][:-5]))):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception:
        continue
    c = d["config"]
    k = d["kernels"].get("gather_reduce") or d["kernels"].get("gat") or {}
    print(f"| {c['workload'].split(':')[0]} | {c['model']} | {c['E_max']} | {d['ms_per_step']:.2f} | {d['value']:.3g} | "
          f"{k.get('ms_per_step', 0):.2f} | {k.get('GB/s') or 0:.0f} | {'/'.join(str(q['items']) for q in c['plans'])} / {'/'.join(str(q['split_rows']) for q in c['plans'])} |")
