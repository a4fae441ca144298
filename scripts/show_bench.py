"""Summarise bench JSON lines: python scripts/show_bench.py gpurun_out/bench_*.json"""
import json
import sys

for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "unreadable", e)
        continue
    r = d["roofline"]
    print(f"{f}: {d['ms_per_step']:.2f} ms/step value={d['value']:.3g} e2e={d['e2e'] and round(d['e2e']['ms_per_step'], 2)} ms "
          f"launches={d['gpu_launches']} roof[{r['class']}] {r['achieved']:.0f} GB/s frac={r['frac']:.2f} share={r['share_of_step']:.2f}")
    for k, v in d["kernels"].items():
        gb = v["GB/s"] and round(v["GB/s"])
        tf = v["TFLOP/s"] and round(v["TFLOP/s"], 1)
        print(f"    {k:14s} {v['ms_per_step']:8.3f} ms x{v['launches_per_step']:.0f}  GB/s {gb}  TF {tf}")
