nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/launch scripts/micro/launch.cu && /tmp/launch | tee gpurun_out/micro_launch_r2.txt
