set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -k "pdl or parity_vs_oracle or full_size" 2>&1 | tail -3
run() { name=$1; shift; timeout 300 python bench.py --steps 2000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'])" || tail -3 gpurun_out/bench_$name.err; }
run base
run base_notiming --no-kernel-timing
run pdl --pdl
run pdl_notiming --pdl --no-kernel-timing
run base2
run pdl2 --pdl
run pdl_r12 --pdl --recon 12
run pdl_f32 --pdl --precision f32
run pdl_48 --pdl --global-dims 48,48,48,48 --steps 300
