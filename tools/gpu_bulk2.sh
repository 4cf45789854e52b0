set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -6
run() { name=$1; shift; python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'])" || tail -3 gpurun_out/bench_$name.err; }
run bulk --kernel bulk
run bulk_r12 --kernel bulk --recon 12
run bulk_f32 --kernel bulk --precision f32
run bulk48 --kernel bulk --global-dims 48,48,48,48 --steps 200
for m in 0.1 0.05; do python tools/bench_cg.py --mass $m; done
python tools/bench_cg.py --mass 0.05 --precision mixed
