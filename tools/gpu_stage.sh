# usage: bash tools/gpu_stage.sh TAG  (GPU box, repo root): staged-kernel tests and benches
TAG=${1:-stage}
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests/test_gpu_stage.py -q --timeout 400 -x 2>&1 | tail -15 > gpurun_out/gpu_tests_$TAG.txt
cat gpurun_out/gpu_tests_$TAG.txt
run() { name=$1; shift; timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/b_${TAG}_$name.json 2> gpurun_out/b_${TAG}_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/b_${TAG}_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'])" || tail -5 gpurun_out/b_${TAG}_$name.err; }
run dir2 --kernel dir2
run dir2_stage --kernel dir2 --stage
run site_stage --kernel site --stage
for n in 2 4 8; do
  run site_n$n --kernel site --nrhs $n
  run site_stage_n$n --kernel site --nrhs $n --stage
  run dir2_stage_n$n --kernel dir2 --nrhs $n --stage
done
run f32_dir2_stage --precision f32 --stage
run f32_site_stage_n8 --precision f32 --kernel site --nrhs 8 --stage
run halo_t_stage --force-halo 8 --stage
echo done
