set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
run() { name=$1; shift; python bench.py --steps 500 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'], 'bnd', r.get('boundary_kernel_us'), d['ms_per_step'])" || tail -3 gpurun_out/bench_$name.err; }
run strong48 --global-dims 48,48,48,48 --steps 200
run selfhalo_t --force-halo 8
run selfhalo_tz --force-halo 12
run selfhalo_t_nooverlap --force-halo 8 --no-overlap
run strong48_selfhalo_t --global-dims 48,48,48,48 --force-halo 8 --steps 200
for m in 0.1 0.05 0.02; do python tools/bench_cg.py --mass $m; done
python tools/bench_cg.py --mass 0.05 --precision mixed
