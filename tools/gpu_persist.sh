set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -8
run() { name=$1; shift; timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'], 'bnd', r.get('boundary_kernel_us'), d['ms_per_step'], d['gpu_launches'])" || tail -3 gpurun_out/bench_$name.err; }
run persist
run classic --no-persistent
run persist_site --kernel site
run persist_dir4 --kernel dir4
run persist_selfhalo_t --force-halo 8
run persist_selfhalo_tz --force-halo 12
run classic_selfhalo_t --force-halo 8 --no-persistent
run persist48 --global-dims 48,48,48,48 --steps 200
run persist48_selfhalo_t --global-dims 48,48,48,48 --force-halo 8 --steps 200
run persist_f32 --precision f32
run persist_r12 --recon 12
run persist_f32r12 --precision f32 --recon 12
for b in 64 128 256; do run persist_b$b --block $b; done
