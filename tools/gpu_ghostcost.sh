# usage: bash tools/gpu_ghostcost.sh: cost of the ghost-aware kernel (all sites through it: overlap none) and the split, 32^4 and 48^3x6
for args in "--force-halo 0" "--force-halo 8 --no-overlap" "--force-halo 8" "--force-halo 8 --overlap fused" "--local 48,48,48,6 --force-halo 0" "--local 48,48,48,6 --force-halo 8 --no-overlap" "--local 48,48,48,6 --force-halo 8"; do
timeout 200 python bench.py $args --steps 1000 --warmup 10 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print('$args |', round(d['ms_per_step']*1e3,1), 'us/step', d['value'], 'GFLOP/s')"
done
