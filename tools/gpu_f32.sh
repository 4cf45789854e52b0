set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1200 python -m pytest tests -m gpu -x -q --timeout 300 -k "precision or recon or roundtrip or multi_rhs or p2p" 2>&1 | tail -3
run() { name=$1; shift; timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'])" || tail -3 gpurun_out/bench_$name.err; }
run f32 --precision f32
run f32_site --precision f32 --kernel site
run f32_dir4 --precision f32 --kernel dir4
run mixed --precision mixed
run f32r12 --precision f32 --recon 12
run f32n4 --precision f32 --nrhs 4 --kernel site
run f32n8 --precision f32 --nrhs 8 --kernel site
run mixedn4 --precision mixed --nrhs 4 --kernel site
