#!/bin/bash
# compute-sanitizer memcheck / racecheck / synccheck over every configuration of
# tools/sanitize_run.py (run on the GPU box from the repo root): bash tools/gpu_sanitize.sh <outdir>
out=${1:-gpurun_out/sanitize}
mkdir -p "$out"
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python tools/sanitize_run.py > "$out/$tool.txt" 2>&1
  echo "$tool rc=$?"; tail -3 "$out/$tool.txt"
done
