#!/bin/bash
# one compute-sanitizer tool per call (TOOL=memcheck|synccheck|racecheck), after a plain run
mkdir -p gpurun_out/r02san
timeout 600 python tools/sanitizer_case.py > gpurun_out/r02san/plain.log 2>&1 || { echo "plain run failed"; tail -5 gpurun_out/r02san/plain.log; exit 1; }
timeout 1500 compute-sanitizer --tool $TOOL --target-processes all python tools/sanitizer_case.py > gpurun_out/r02san/sanitizer_$TOOL.log 2>&1
echo "$TOOL rc=$? $(tail -1 gpurun_out/r02san/sanitizer_$TOOL.log)"; grep -c "Error\|Hazard" gpurun_out/r02san/sanitizer_$TOOL.log
