set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 900 python -m pytest tests/test_gpu_parity.py -x -q -k "bulk" 2>&1 | tail -8
run() { name=$1; shift; python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'], 'bnd', r.get('boundary_kernel_us'), d['ms_per_step'])" || tail -3 gpurun_out/bench_$name.err; }
run bulk --kernel bulk
run dir2 --kernel dir2
run bulk_r12 --kernel bulk --recon 12
run bulk_f32 --kernel bulk --precision f32
run bulk48 --kernel bulk --global-dims 48,48,48,48 --steps 200
run selfhalo_t_nooverlap --force-halo 8 --no-overlap
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dslash_bulk -s 5 -c 1 \
    -o gpurun_out/prof_bulk -f python bench.py --kernel bulk --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_bulk.log 2>&1
tail -2 gpurun_out/ncu_bulk.log
