# usage: bash tools/gpu_r9sweep.sh [recon]: launch-configuration sweep at 32^4 fp64 (bench.py, 300 steps)
mkdir -p gpurun_out
R=${1:-9}
for k in dir2 site; do for b in 64 128 256; do for m in 2 3; do
timeout 120 python bench.py --recon $R --kernel $k --block $b --min-blocks $m --steps 300 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print('recon $R', '$k', $b, $m, d['value'], round(d['ms_per_step']*1e3,1), d['roofline']['frac'])"
done; done; done
