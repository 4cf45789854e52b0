python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_blocked.py tests/test_gpu_full_size.py -q -x -k "blocked or multi_rhs" 2>&1 | tail -3
run() { timeout 300 python bench.py --steps 500 --warmup 20 --no-cpu-baseline --no-e2e --no-read-calibration "$@" 2>/tmp/err.txt | python -c "import json,sys; d=json.loads(sys.stdin.readline()); r=d['roofline']; print('%-50s %10.2f %7.4f %8.2f us' % (' '.join(sys.argv[1:]), d['value'], r['frac'], r['avg_launch_us']))" "$@" || tail -2 /tmp/err.txt; }
for rep in 1 2; do
for p in f64 f32 mixed; do for n in 8 4 2; do
  run --nrhs $n --precision $p
  run --nrhs $n --precision $p --layout blocked
done; done
run --nrhs 8 --recon 12; run --nrhs 8 --recon 12 --layout blocked
run --nrhs 8 --recon 9; run --nrhs 8 --recon 9 --layout blocked
done
