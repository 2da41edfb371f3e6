nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/micro scripts/micro/micro.cu && /tmp/micro | tee gpurun_out/micro_r2.txt
