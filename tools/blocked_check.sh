# site-blocked layout: tests + bench lines (planar vs blocked) on one box
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1500 python -m pytest tests/test_gpu_blocked.py tests/test_gpu_multiproc.py tests/test_gpu_full_size.py -q -x -k "blocked" 2>&1 | tail -3
run() { timeout 300 python bench.py --steps 500 --warmup 20 --no-cpu-baseline --no-e2e --no-read-calibration "$@" 2>/tmp/err.txt | python -c "import json,sys; d=json.loads(sys.stdin.readline()); r=d['roofline']; print('%-52s %10.2f %7.4f %8.2f us' % (' '.join(sys.argv[1:]), d['value'], r['frac'], r['avg_launch_us']))" "$@" || tail -2 /tmp/err.txt; }
for rep in 1 2; do
for a in "" "--precision f32" "--precision mixed" "--recon 12" "--recon 9" "--precision mixed --recon 12"; do
  run --nrhs 8 $a; run --nrhs 8 --layout blocked $a
done
run --nrhs 8 --layout blocked --force-halo 8; run --nrhs 8 --force-halo 8
run --nrhs 8 --layout blocked --force-halo 12; run --nrhs 8 --force-halo 12
done
