set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
run() { name=$1; shift; timeout 300 python bench.py --steps 300 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'])" || tail -3 gpurun_out/bench_$name.err; }
run strong_t8_local --local 48,48,48,6 --force-halo 8
run strong_t4_local --local 48,48,48,12 --force-halo 8
run strong_t2_local --local 48,48,48,24 --force-halo 8
run strong_t4z2_local --local 48,48,24,12 --force-halo 12
run strong_t8_nohalo --local 48,48,48,6
run strong_t8_local_site --local 48,48,48,6 --force-halo 8 --kernel site
run strong_t8_local_dir4 --local 48,48,48,6 --force-halo 8 --kernel dir4
