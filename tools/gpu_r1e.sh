# usage: bash tools/gpu_r1e.sh: re-entry check after a container rebuild: smoke, full GPU suite, default bench
set -x
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
timeout 600 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -2
timeout 2400 python -m pytest tests -m gpu -q --timeout 600 -x 2>&1 | tail -8 > gpurun_out/gpu_tests_r1e.txt
cat gpurun_out/gpu_tests_r1e.txt
timeout 600 python bench.py > gpurun_out/bench_r1e.json 2> gpurun_out/bench_r1e.err; cat gpurun_out/bench_r1e.json
echo done
