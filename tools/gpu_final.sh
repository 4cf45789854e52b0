#!/bin/bash
# End-of-round evidence on one GPU box (from the repo root): bash tools/gpu_final.sh <name>
# (compute-sanitizer is closed on this pool: tools/gpu_sanitize.sh is run separately where it is open;
# the .ncu-rep files are deleted after their CSV export: gpurun copies back at most 64 MiB)
n=${1:-r03_final}
bash tools/gpu_run.sh $n \
  "timeout 2400 python -m pytest tests -m gpu -q --timeout 900" \
  "timeout 300 python -c 'import __graft_entry__ as g; g.smoke()'" \
  "timeout 300 python bench.py --steps 20 --warmup 5" \
  "timeout 300 python bench.py --no-cpu-baseline" \
  "timeout 600 python bench.py --impl reference --steps 20 --warmup 5" \
  "bash tools/gpu_ncu.sh gpurun_out/$n/ncu_headline" \
  "bash tools/gpu_ncu.sh gpurun_out/$n/ncu_n8 --nrhs 8" \
  "bash tools/gpu_ncu.sh gpurun_out/$n/ncu_n8_blocked --nrhs 8 --layout blocked" \
  "bash tools/gpu_ncu.sh gpurun_out/$n/ncu_n8_f32_blocked --nrhs 8 --layout blocked --precision f32" \
  "bash tools/config_table.sh" \
  "bash tools/halo_probe.sh" \
  "bash tools/strong_probe.sh" \
  "timeout 600 python tools/bench_cg_multi.py" \
  "timeout 300 python bench.py --nrhs 8 --layout blocked --no-cpu-baseline" \
  "timeout 300 python bench.py --nrhs 8 --layout blocked --precision f32 --no-cpu-baseline" \
  "find gpurun_out/$n -name '*.ncu-rep' -delete"
