# usage: bash tools/gpu_fused2.sh TAG: fused-mode re-measure + serialised launch lists of the overlap modes
TAG=${1:-f2}
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 600 python -m pytest tests/test_gpu_overlap_fused.py -q --timeout 300 -x 2>&1 | tail -3
run() { name=$1; shift; timeout 300 python bench.py --steps 1000 --no-cpu-baseline --no-e2e "$@" > gpurun_out/b_${TAG}_$name.json 2> gpurun_out/b_${TAG}_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/b_${TAG}_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'], d['gpu_launches'])" 2>/dev/null || tail -3 gpurun_out/b_${TAG}_$name.err; }
run t_fused --force-halo 8 --overlap fused
run t_fused_nccl --force-halo 8 --overlap fused --self-nccl
run t_sites_nccl --force-halo 8 --self-nccl
run t8_fused --local 48,48,48,6 --force-halo 8 --overlap fused
run t4z2_fused --local 48,48,24,12 --force-halo 12 --overlap fused
run t4z2_sites --local 48,48,24,12 --force-halo 12
for m in sites fused none; do
  timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ncu_${TAG}_$m.csv python bench.py --steps 4 --warmup 3 --no-cpu-baseline --no-e2e --force-halo 8 $( [ $m = none ] && echo --no-overlap || echo --overlap $m ) > /dev/null 2>&1
  python - <<PY
import csv
rows=[r for r in csv.reader(open('gpurun_out/ncu_${TAG}_$m.csv')) if len(r) > 14 and r[12] == 'gpu__time_duration.sum']
for r in rows[-12:]: print('$m', r[4][:60], r[8], r[14])
PY
done
echo done
