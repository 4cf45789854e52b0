set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
run() { name=$1; shift; python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['clocks'])" || tail -3 gpurun_out/bench_$name.err; }
run r12 --recon 12
run n2 --nrhs 2
run n4 --nrhs 4
run n8 --nrhs 8
run f32r12 --precision f32 --recon 12
run f32n4 --precision f32 --nrhs 4
run n4r12 --nrhs 4 --recon 12
run site --kernel site
