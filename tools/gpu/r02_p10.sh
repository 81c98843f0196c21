#!/bin/bash
mkdir -p gpurun_out/r02p
nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o /tmp/probe10 probes/probe10.cu && /tmp/probe10 > gpurun_out/r02p/probe10.jsonl
cat gpurun_out/r02p/probe10.jsonl
