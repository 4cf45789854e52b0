# usage: bash tools/gpu_sanitize2.sh: compute-sanitizer memcheck / racecheck / synccheck over every
# configuration of tools/sanitize_run.py (26: + producer push, recon-9)
mkdir -p gpurun_out
for tool in memcheck racecheck synccheck; do
  timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python tools/sanitize_run.py > gpurun_out/sanitize2_$tool.txt 2>&1
  echo "$tool rc=$?"; tail -3 gpurun_out/sanitize2_$tool.txt
done
