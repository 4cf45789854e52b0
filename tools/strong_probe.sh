# 48^4 strong-scaling per-GPU volumes on one GPU (self-halo proxy), event-free steps:
# bash tools/strong_probe.sh
B="python bench.py --steps 1000 --warmup 50 --no-cpu-baseline --no-e2e --no-read-calibration --breakdown-steps 100"
run() { timeout 300 $B "$@" 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.readline()); b=(d['roofline'].get('breakdown') or {})
print('%-62s %8.2f us/step  frac %.3f  span %s  int %s  bnd %s  exch %s' % (' '.join(sys.argv[1:]), d['ms_per_step']*1e3, d['roofline']['frac'], b.get('span_us'), b.get('interior_us'), b.get('boundary_us'), b.get('exchange_us')))" "$@"; }
run --local 48,48,48,6
run --local 48,48,48,6 --force-halo 8
run --local 48,48,48,6 --force-halo 8 --overlap dirs
run --local 48,48,48,6 --force-halo 8 --no-overlap
run --local 48,48,48,6 --force-halo 8 --transport p2p
run --local 48,48,48,6 --force-halo 8 --transport p2p --overlap dirs
run --local 48,48,24,12
run --local 48,48,24,12 --force-halo 12
run --local 48,48,24,12 --force-halo 12 --transport p2p
run --local 48,48,48,12
run --local 48,48,48,12 --force-halo 8
run --local 48,48,48,24 --force-halo 8
