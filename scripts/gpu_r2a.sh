set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests/test_gpu_stack.py tests/test_gpu_conv_rgcn.py -m gpu -q -x > gpurun_out/gputest3.log 2>&1
echo rc=$? >> gpurun_out/gputest3.log
timeout 600 python bench.py --config C5 --rank-slice 8 --steps 5 --warmup 3 > gpurun_out/bench_c5slice.json 2> gpurun_out/bench_c5slice.err
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/bench_c4.json 2> gpurun_out/bench_c4.err
cd scripts && nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gran_probe gran_probe.cu && ./gran_probe > ../gpurun_out/gran.txt 2>&1
timeout 300 ncu --metrics dram__bytes_read.sum,gpu__time_duration.sum --csv ./gran_probe > ../gpurun_out/gran_ncu.csv 2>&1
