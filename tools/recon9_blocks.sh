run() { timeout 600 python bench.py --steps 1000 --warmup 50 --no-cpu-baseline --no-e2e --no-read-calibration "$@" 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.readline()); r=d['roofline']
print('%-50s %9.1f %7.2f us %.3f' % (' '.join(sys.argv[1:]), d['value'], d['ms_per_step']*1e3, r['frac']))" "$@"; }
for p in f64 f32 mixed; do for b in 64 128 256; do run --recon 9 --precision $p --block $b; run --recon 9 --precision $p --block $b --kernel dir2; done; done
for b in 64 128 256; do run --precision mixed --block $b; run --precision mixed --recon 12 --block $b; done
