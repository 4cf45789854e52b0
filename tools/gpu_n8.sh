set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -k "multi_rhs" 2>&1 | tail -3
run() { name=$1; shift; timeout 300 python bench.py --steps 500 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'])" || tail -3 gpurun_out/bench_$name.err; }
for k in site dir2 dir4; do run ${k}_n8 --nrhs 8 --kernel $k; done
run f32_n8 --nrhs 8 --kernel site --precision f32
run r12_n8 --nrhs 8 --kernel site --recon 12
