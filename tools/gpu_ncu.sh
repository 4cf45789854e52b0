#!/bin/bash
# ncu evidence for one bench configuration (run on the GPU box, from the repo root):
#   bash tools/gpu_ncu.sh <outdir> [bench.py args...]
# 1. launch list: gpu__time_duration of every kernel of a short bench run (the recipe's
#    --clock-control none pass; per-launch times are cold-cache and serialised),
# 2. one `ncu --set full --import-source on` capture of the 6th stencil launch, exported as
#    details / raw CSV next to the .ncu-rep.
out=$1; shift
mkdir -p "$out"
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file "$out/launches.csv" \
  python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-read-calibration "$@" > "$out/launches_bench.txt" 2>&1
echo "launch list rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dslash -s 5 -c 1 -o "$out/full" -f \
  python bench.py --steps 8 --warmup 3 --no-cpu-baseline --no-e2e --no-read-calibration "$@" > "$out/full_bench.txt" 2>&1
echo "full capture rc=$?"
ncu -i "$out/full.ncu-rep" --page details --csv > "$out/full_details.csv" 2>&1
ncu -i "$out/full.ncu-rep" --page raw --csv > "$out/full_raw.csv" 2>&1
