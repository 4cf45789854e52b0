python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 python bench.py --steps 300 --warmup 20 --no-cpu-baseline --no-e2e --no-read-calibration "$@" 2>/tmp/err.txt | python -c "import json,sys; d=json.loads(sys.stdin.readline()); r=d['roofline']; import math; print('%-50s %10.2f %7.4f %8.2f us' % (' '.join(sys.argv[1:]), d['value'], r['frac'], r['avg_launch_us']))" "$@" || tail -2 /tmp/err.txt; }
for rep in 1 2; do
for L in 32,32,32,32 32,32,32,30 32,32,32,28 32,32,32,36 32,32,30,32 48,48,48,24; do
  run --local $L --nrhs 8 --precision f32
  run --local $L --nrhs 8
done
done
