# usage: bash tools/gpu_mrhs_block.sh: block-size sweep of the multi-RHS kernels (L1 locality of y hops)
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for n in 8 4 2; do for k in site dir2; do for b in 64 128 256; do
  timeout 300 python bench.py --steps 500 --warmup 20 --no-cpu-baseline --no-e2e --kernel $k --nrhs $n --block $b > gpurun_out/mb_${k}_n${n}_b$b.json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/mb_${k}_n${n}_b$b.json')); r=d['roofline']
print('$k n=$n block=$b', d['value'], 'frac', r['frac'], 'us', r['avg_launch_us'], 'clk', d['clocks']['sm_mhz'])" 2>/dev/null
done; done; done
echo done
