import json, sys
for f in sys.argv[1:]:
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
    except Exception as e:
        print(f, "ERR", e); continue
    print(f, "ms", round(d["ms_per_step"], 3), "value %.3e" % d["value"], "frac", round(d["roofline"]["frac"], 3),
          d["config"].get("launch_mode"), d["config"].get("graph_capture_error"))
    print("  ", {k: (round(v["ms_per_step"], 3), v["launches_per_step"], round(v["GB/s"] or 0)) for k, v in d["kernels"].items()})
    if d.get("step_time"): print("   step", {k: (round(v, 3) if isinstance(v, float) else v) for k, v in d["step_time"].items()})
    if d.get("per_layer"): print("   layers", [(p["layer"], round(p["fwd_ms"], 3), round(p["bwd_ms"], 3)) for p in d["per_layer"]])
    if d.get("e2e"): print("   e2e", round(d["e2e"]["ms_per_step"], 3))
