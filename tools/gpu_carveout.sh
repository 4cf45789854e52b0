# usage: bash tools/gpu_carveout.sh: stencil throughput vs the shared-memory carveout preference (HISQ_L1_CARVEOUT)
for cv in default 0 50 100; do
for args in "--kernel dir2" "--kernel site --nrhs 8" "--kernel site --nrhs 4" "--kernel site --nrhs 8 --precision f32"; do
if [ $cv = default ]; then unset HISQ_L1_CARVEOUT; else export HISQ_L1_CARVEOUT=$cv; fi
timeout 200 python bench.py $args --steps 500 --warmup 10 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print('carveout $cv | $args |', round(d['ms_per_step']*1e3,1), 'us', d['value'], d['roofline']['frac'])"
done; done
