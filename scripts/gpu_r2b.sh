mkdir -p gpurun_out
cd scripts && nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o gran_probe gran_probe.cu && ./gran_probe > ../gpurun_out/gran2.txt 2>&1
timeout 300 ncu --metrics dram__bytes_read.sum --csv ./gran_probe > ../gpurun_out/gran2_ncu.csv 2>&1
