# usage: bash tools/gpu_final5.sh: sanitizer sweep (memcheck / racecheck / synccheck) over
# tools/sanitize_run.py and the ncu launch list of the default bench command, current build
mkdir -p gpurun_out/final5
for tool in memcheck racecheck synccheck; do
  timeout 900 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python tools/sanitize_run.py > gpurun_out/final5/sanitize_$tool.txt 2>&1
  echo "$tool rc=$?" | tee -a gpurun_out/final5/sanitize_rc.txt; tail -2 gpurun_out/final5/sanitize_$tool.txt
done
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/final5/launches.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
echo "ncu rc=$?"
