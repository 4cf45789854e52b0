# usage: bash tools/gpu_check.sh  (runs on the GPU box from the repo root)
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
nproc; free -g | head -2
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -5
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -15 > gpurun_out/gpu_tests.txt
cat gpurun_out/gpu_tests.txt
for k in site dir4; do
  timeout 600 python bench.py --kernel $k --steps 1000 --warmup 20 --no-cpu-baseline > gpurun_out/bench_$k.json 2> gpurun_out/bench_$k.err
  tail -2 gpurun_out/bench_$k.err; cat gpurun_out/bench_$k.json
done
