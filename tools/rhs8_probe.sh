run() { timeout 300 env $1 python bench.py --steps 300 --warmup 10 --no-cpu-baseline --no-e2e --no-read-calibration --nrhs 8 $2 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); r=d['roofline']; print('$1 $2', d['value'], r['frac'], r['avg_launch_us'])"; }
run X=0 --no-rhs8-tma
run HISQ_RHS8_UNROLL=1 ""
run HISQ_RHS8_UNROLL=4 ""
for u in 1 4; do HISQ_RHS8_UNROLL=$u timeout 600 python -m pytest tests/test_gpu_parity.py -q -x -k rhs8 2>&1 | tail -1; done
