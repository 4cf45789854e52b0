set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 900 python -m pytest tests -m gpu -x -q --timeout 300 -k "timing or halo" 2>&1 | tail -3
run() { name=$1; shift; timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'algoGB/s', d['algorithmic_gbs'], 'frac', r['frac'], 'us', r['avg_launch_us'], r['kernel'], d['ms_per_step'])" || tail -3 gpurun_out/bench_$name.err; }
run span_selfhalo_t --force-halo 8
run span_selfhalo_tz --force-halo 12
run span_48_selfhalo_t --global-dims 48,48,48,48 --force-halo 8 --steps 200
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29531 \
     bench.py --gpus 2 --colocate --steps 50 --warmup 3 --no-e2e > gpurun_out/bench_colocate_span.json 2> gpurun_out/bench_colocate_span.err
echo rc=$?; python -c "import json; d=json.load(open('gpurun_out/bench_colocate_span.json')); print(d['roofline'])"
