#!/bin/bash
mkdir -p gpurun_out
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/fp64_mix tools/ubench/fp64_mix.cu && /tmp/fp64_mix > gpurun_out/r02t_fp64_mix.jsonl; cat gpurun_out/r02t_fp64_mix.jsonl
nvidia-smi --query-gpu=clocks.sm,clocks.max.sm,power.draw --format=csv
