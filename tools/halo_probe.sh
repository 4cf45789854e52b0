# Halo-overhead decomposition on one GPU (self-halo), event-free timed region, 1000 steps each:
# bash tools/halo_probe.sh > out.txt
B="python bench.py --steps 1000 --warmup 50 --no-cpu-baseline --no-e2e --no-read-calibration --breakdown-steps 100"
run() { timeout 300 $B "$@" 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.readline()); b=(d['roofline'].get('breakdown') or {})
print('%-45s %8.2f us/step  span %s  int %s  bnd %s  exch %s' % (' '.join(sys.argv[1:]), d['ms_per_step']*1e3, b.get('span_us'), b.get('interior_us'), b.get('boundary_us'), b.get('exchange_us')))" "$@"; }
for i in 1 2; do
run
run --no-pdl
run --force-halo 8
run --force-halo 8 --halo-dryrun
run --force-halo 8 --no-overlap
run --force-halo 8 --no-pdl
run --force-halo 12
run --force-halo 12 --halo-dryrun
run --force-halo 12 --no-overlap
run --force-halo 8 --transport p2p
run --force-halo 12 --transport p2p
done
