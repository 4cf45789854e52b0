set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15
run() { name=$1; shift; python bench.py --steps 500 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'])" || tail -3 gpurun_out/bench_$name.err; }
for k in dir2 site dir4; do for n in 2 4 8; do run ${k}_n$n --nrhs $n --kernel $k; done; done
run n4r12 --nrhs 4 --recon 12
run f32n4 --precision f32 --nrhs 4
run f32n8 --precision f32 --nrhs 8
