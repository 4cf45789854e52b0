# usage: bash tools/gpu_fused.sh TAG  (GPU box, repo root): one-shot fused overlap tests and benches
TAG=${1:-fused}
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_overlap_fused.py tests/test_gpu_multiproc.py -q --timeout 300 -x -k "fused" 2>&1 | tail -15 > gpurun_out/gpu_tests_$TAG.txt
cat gpurun_out/gpu_tests_$TAG.txt
run() { name=$1; shift; timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/b_${TAG}_$name.json 2> gpurun_out/b_${TAG}_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/b_${TAG}_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'])" 2>/dev/null || tail -3 gpurun_out/b_${TAG}_$name.err; }
run nohalo
run t_sites --force-halo 8
run t_fused --force-halo 8 --overlap fused
run t_fused_nccl --force-halo 8 --overlap fused --self-nccl
run t_fused_p2p --force-halo 8 --overlap fused --transport p2p
run t_sites_nccl --force-halo 8 --self-nccl
run tz_sites --force-halo 12
run tz_fused --force-halo 12 --overlap fused
run t8_sites --local 48,48,48,6 --force-halo 8
run t8_fused --local 48,48,48,6 --force-halo 8 --overlap fused
run t4_fused --local 48,48,48,12 --force-halo 8 --overlap fused
run t4z2_fused --local 48,48,24,12 --force-halo 12 --overlap fused
python tools/probe_overlap.py 32,32,32,32 8 2>&1 | tail -8
echo done
