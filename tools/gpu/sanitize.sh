#!/bin/bash
mkdir -p gpurun_out/r02san
for tool in memcheck racecheck synccheck; do
  timeout 1200 compute-sanitizer --tool $tool --target-processes all python tools/sanitizer_case.py > gpurun_out/r02san/sanitizer_$tool.log 2>&1
  echo "$tool rc=$? $(tail -1 gpurun_out/r02san/sanitizer_$tool.log)"
done
