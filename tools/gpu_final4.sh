# usage: bash tools/gpu_final4.sh: final evidence after the CG fusion: memcheck + racecheck over the
# sanitizer configurations, smoke, full GPU suite, default bench
mkdir -p gpurun_out/final4
for tool in memcheck racecheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python tools/sanitize_run.py > gpurun_out/final4/sanitize_$tool.txt 2>&1
  echo "$tool rc=$?"; tail -2 gpurun_out/final4/sanitize_$tool.txt
done
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1 > gpurun_out/final4/smoke.txt
timeout 2400 python -m pytest tests -m gpu -q --timeout 600 2>&1 | tail -4 > gpurun_out/final4/gpu_tests.txt
timeout 600 python bench.py > gpurun_out/final4/bench.json 2> gpurun_out/final4/bench.err
cat gpurun_out/final4/smoke.txt gpurun_out/final4/gpu_tests.txt gpurun_out/final4/bench.json
