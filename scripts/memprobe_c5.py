import sys, os, time, numpy as np, torch
sys.path.insert(0, os.getcwd())
import synth, paper_conf_eurosys_huangz0wjzzzys24_b200 as wg
from paper_conf_eurosys_huangz0wjzzzys24_b200.stack import partition_1d
c = synth.CONFIGS["C5"]
block, bounds = partition_1d(c.V, 8)
vb, ve = bounds[0]
t0 = time.time()
src, dst = synth.make_graph_slice(c.V, c.E, vb, ve, seed=c.seed * 16, alpha=c.alpha)
print("slice", len(src), time.time() - t0, flush=True)
g = wg.Graph(torch.from_numpy(src).cuda(), torch.from_numpy(dst).cuda(), num_vertices=c.V, v_begin=vb, v_end=ve)
torch.cuda.synchronize()
print("graph mem GB", torch.cuda.memory_allocated() / 1e9, "E_fwd", g.E_fwd, "E_T", g.E_T, flush=True)
fi = [128, 32, 32]
for i, fo in enumerate([32, 32, 172]):
    cv = wg.Conv(g, "sage", fi[i], fo, dtype=torch.bfloat16, fuse_relu=i < 2, need_dx=i > 0)
    print(f"layer {i}: ws {cv.ws_bytes/1e9:.2f} GB saved {cv.saved_bytes/1e9:.2f} GB edge {cv.n_edge_tasks} vert {cv.n_vertex_tasks} bwd_path {cv.bwd_path}", flush=True)
    del cv
    torch.cuda.empty_cache()
