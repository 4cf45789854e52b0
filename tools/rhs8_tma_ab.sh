python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 env $1 python bench.py --steps 500 --warmup 20 --no-cpu-baseline --no-e2e --no-read-calibration $2 2>/tmp/err.txt | python -c "import json,sys; d=json.loads(sys.stdin.readline()); r=d['roofline']; print('%-20s %-30s %10.2f %7.4f %8.2f us' % (sys.argv[1], sys.argv[2], d['value'], r['frac'], r['avg_launch_us']))" "$1" "$2" || tail -3 /tmp/err.txt; }
for rep in 1 2 3; do
  for v in X=0 HISQ_RHS8_TMA=0 HISQ_RHS8_TMA=1 HISQ_RHS8_TMA=2 HISQ_RHS8_TMA=3; do run $v "--nrhs 8"; done
done
run HISQ_RHS8_TMA=0 "--nrhs 8 --recon 12"; run X=0 "--nrhs 8 --recon 12"
HISQ_RHS8_TMA=0 timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_full_size.py -q -x -k "multi_rhs or rhs8" 2>&1 | tail -3
