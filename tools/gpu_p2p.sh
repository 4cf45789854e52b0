set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -3
timeout 1800 python -m pytest tests -m gpu -x -q --timeout 300 --timeout-method thread 2>&1 | tail -15
run() { name=$1; shift; timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'], d['gpu_launches'])" || tail -3 gpurun_out/bench_$name.err; }
run persist_always --persistent-always
run classic --no-persistent
run persist_selfhalo_t --force-halo 8
run classic_selfhalo_t --force-halo 8 --no-persistent
run persist_selfhalo_tz --force-halo 12
run persist48 --global-dims 48,48,48,48 --steps 200
run persist_f32 --precision f32
run persist_r12 --recon 12
