# usage: bash tools/gpu_dirs.sh TAG  (GPU box, repo root): split-by-direction overlap tests and benches
TAG=${1:-dirs}
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python -m pytest tests/test_gpu_overlap_dirs.py tests/test_gpu_multiproc.py -q --timeout 600 -x -k "dirs" 2>&1 | tail -15 > gpurun_out/gpu_tests_$TAG.txt
cat gpurun_out/gpu_tests_$TAG.txt
run() { name=$1; shift; timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/b_${TAG}_$name.json 2> gpurun_out/b_${TAG}_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/b_${TAG}_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'])" || tail -5 gpurun_out/b_${TAG}_$name.err; }
run nohalo
run t_sites --force-halo 8
run t_dirs --force-halo 8 --overlap dirs
run t_dirs_nccl --force-halo 8 --overlap dirs --self-nccl
run tz_sites --force-halo 12
run tz_dirs --force-halo 12 --overlap dirs
run t8_sites --local 48,48,48,6 --force-halo 8
run t8_dirs --local 48,48,48,6 --force-halo 8 --overlap dirs
run t8_none --local 48,48,48,6 --force-halo 8 --no-overlap
run t4_sites --local 48,48,48,12 --force-halo 8
run t4_dirs --local 48,48,48,12 --force-halo 8 --overlap dirs
run t4z2_sites --local 48,48,24,12 --force-halo 12
run t4z2_dirs --local 48,48,24,12 --force-halo 12 --overlap dirs
echo done
