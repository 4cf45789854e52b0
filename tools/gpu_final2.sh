set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -3
timeout 2400 python -m pytest tests -m gpu -q --timeout 400 2>&1 | tail -5
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > gpurun_out/clocks_final2.csv &
SMI=$!
timeout 600 python bench.py > gpurun_out/bench_final2.json 2> gpurun_out/bench_final2.err
kill $SMI
cat gpurun_out/bench_final2.json; tail -2 gpurun_out/bench_final2.err
run() { name=$1; shift; timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'])" || tail -3 gpurun_out/bench_$name.err; }
run r12 --recon 12
run f32 --precision f32
run f32r12 --precision f32 --recon 12
run mixed --precision mixed
run n2 --nrhs 2 --kernel site
run n4 --nrhs 4 --kernel site
run n8 --nrhs 8 --kernel site
run f32n8 --nrhs 8 --kernel site --precision f32
run strong48 --global-dims 48,48,48,48 --steps 300
run selfhalo_t --force-halo 8
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_final2.csv \
    python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
echo done
