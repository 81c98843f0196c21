#!/bin/bash
mkdir -p gpurun_out/r02s
timeout 600 python bench.py --config slicing > gpurun_out/r02s/slicing.json 2> gpurun_out/r02s/slicing.err; echo "slicing rc=$?"; tail -c 800 gpurun_out/r02s/slicing.err
