# Env-knob A/B of the halo split on one GPU (self-halo, event-free timed region, 1000 steps):
#   bash tools/halo_ab.sh "ENV=1" "ENV2=1" ...      (X=0 is the default)
B="python bench.py --steps 1000 --warmup 50 --no-cpu-baseline --no-e2e --no-read-calibration --breakdown-steps 0"
run() { e=$1; shift; timeout 300 env $e $B "$@" 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.readline())
print('%-26s %-40s %8.2f us/step' % (sys.argv[1], ' '.join(sys.argv[2:]), d['ms_per_step']*1e3))" "$e" "$@"; }
for rep in 1 2 3; do
  run X=0
  for e in X=0 "$@"; do
    for a in "--force-halo 8" "--force-halo 12" "--force-halo 8 --transport p2p" "--force-halo 12 --transport p2p"; do run "$e" $a; done
  done
done
