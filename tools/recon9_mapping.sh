# 1-RHS mapping A/B (site vs dir2) per precision and recon at 32^4: bash tools/recon9_mapping.sh
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
run() { timeout 300 python bench.py --steps 1000 --warmup 50 --no-cpu-baseline --no-e2e --no-read-calibration "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); r=d['roofline']; print('%-52s %10.2f %7.4f %8.2f us' % (' '.join(sys.argv[1:]), d['value'], r['frac'], r['avg_launch_us']))" "$@"; }
for rep in 1 2 3; do
for a in "--precision mixed" "--precision mixed --recon 12" "--precision f32 --recon 12" "--recon 12" "--precision f32" ""; do
  run $a --kernel dir2
  run $a --kernel site
done
done
