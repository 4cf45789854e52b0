#!/bin/bash
# Parameterised GPU-box driver (one script instead of per-session ones):
#   bash tools/gpu_run.sh <name> "<command 1>" "<command 2>" ...
# builds everything in-tree (sm_100a), then runs each command from the repo root with its
# stdout+stderr in gpurun_out/<name>/NN.txt and a summary line (rc, seconds) in
# gpurun_out/<name>/summary.txt.  Used as: gpurun -- bash tools/gpu_run.sh r02_x "python bench.py ..."
name=$1; shift
out=gpurun_out/$name
mkdir -p "$out"
python -c "import __graft_entry__ as g; g.build()" > "$out/build.txt" 2>&1 || { echo "build failed"; tail -30 "$out/build.txt"; exit 1; }
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,clocks.mem,power.draw --format=csv > "$out/gpu.txt" 2>&1
i=0
for cmd in "$@"; do
  i=$((i+1)); f=$(printf "%s/%02d.txt" "$out" $i)
  echo "\$ $cmd" > "$f"
  t0=$(date +%s%N)
  bash -c "$cmd" >> "$f" 2>&1
  rc=$?
  t1=$(date +%s%N)
  printf "%02d rc=%d %ds %s\n" $i $rc $(( (t1 - t0) / 1000000000 )) "$cmd" | tee -a "$out/summary.txt"
  tail -3 "$f"
done
