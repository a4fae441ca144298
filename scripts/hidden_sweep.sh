# Fig 20-style hidden-dimension sweep of the distributed layer placement (f3):
# one rank of the 8-way C4 partition (edge-balanced) with the emulated exchange;
# the JSON lines record each layer's plan (EDGE / VERTEX) and exchanged widths.
mkdir -p gpurun_out/sweep
for h in 16 32 64 128 256 512; do
  timeout 600 python bench.py --rank-slice 8 --emulate-xchg --hidden $h --steps 5 --warmup 2 > gpurun_out/sweep/h$h.json 2> gpurun_out/sweep/h$h.err
done
