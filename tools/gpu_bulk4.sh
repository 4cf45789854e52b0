set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 300 -k "bulk or precision or roundtrip or pdl" 2>&1 | tail -3
for tool in racecheck memcheck; do
  timeout 1200 compute-sanitizer --tool $tool --error-exitcode 9 --print-limit 20 python tools/sanitize_run.py > gpurun_out/sanitize_$tool.txt 2>&1
  echo "$tool rc=$?"; tail -2 gpurun_out/sanitize_$tool.txt
done
run() { name=$1; shift; timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'])" || tail -3 gpurun_out/bench_$name.err; }
run bulk --kernel bulk
run bulk_f32 --kernel bulk --precision f32
run bulk_r12 --kernel bulk --recon 12
run bulk48 --kernel bulk --global-dims 48,48,48,48 --steps 200
run bulk_selfhalo --kernel bulk --force-halo 8
