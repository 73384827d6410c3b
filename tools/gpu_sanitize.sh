#!/bin/bash
# compute-sanitizer passes over tools/sanitize_run.py (run inside gpurun).
# Logs go to gpurun_out/<tag>_sanitize_<tool>.log.  Usage: bash tools/gpu_sanitize.sh <tag>
TAG=${1:-san}
mkdir -p gpurun_out
for tool in memcheck synccheck initcheck racecheck; do
  extra=""
  # leak check off: the only leaks reported are torch caching-allocator blocks (r2a log)
  timeout 900 compute-sanitizer --tool $tool $extra --error-exitcode 9 --print-limit 50 \
    python tools/sanitize_run.py > gpurun_out/${TAG}_sanitize_${tool}.log 2>&1
  echo "$tool exit $?" | tee -a gpurun_out/${TAG}_sanitize_${tool}.log
done
