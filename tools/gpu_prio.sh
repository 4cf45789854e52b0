set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
run() { name=$1; shift; timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'], 'bnd', r.get('boundary_kernel_us'), d['ms_per_step'])" || tail -3 gpurun_out/bench_$name.err; }
run prio_selfhalo_t --force-halo 8
run prio_selfhalo_tz --force-halo 12
run prio_selfhalo_t_p2p --force-halo 8 --transport p2p
run prio_48_selfhalo_t --global-dims 48,48,48,48 --force-halo 8 --steps 200
run prio_nohalo
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -k "halo or multirank" 2>&1 | tail -3
