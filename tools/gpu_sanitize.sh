#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over tools/sanitize.py
# (C1 vEB, C1 + CTA-kernel allocator rounds, a serialized replay, a small graph).
mkdir -p gpurun_out
PARTS=${1:-all}
for tool in memcheck racecheck synccheck; do
  extra=""
  [ $tool = memcheck ] && extra="--leak-check no"
  [ $tool = racecheck ] && extra="--racecheck-report all"
  timeout 1500 compute-sanitizer --tool $tool $extra --print-limit 50 \
      python tools/sanitize.py $PARTS > gpurun_out/sanitize_$tool.log 2>&1
  echo "$tool rc=$?"; tail -4 gpurun_out/sanitize_$tool.log
done
