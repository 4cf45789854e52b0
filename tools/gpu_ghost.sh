set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -k "halo or multirank or bulk" 2>&1 | tail -3
run() { name=$1; shift; timeout 300 python bench.py --steps 300 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'])" || tail -3 gpurun_out/bench_$name.err; }
run strong_t8_local --local 48,48,48,6 --force-halo 8
run strong_t8_local_nooverlap --local 48,48,48,6 --force-halo 8 --no-overlap
run strong_t4z2_local --local 48,48,24,12 --force-halo 12
run selfhalo_t --force-halo 8
run nohalo
