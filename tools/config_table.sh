# One bench line per configuration of the published table (32^4 and 48^4, 1 GPU, event-free
# timed region, 1000 steps): bash tools/config_table.sh > table.txt
run() { timeout 600 python bench.py --steps 1000 --warmup 50 --no-cpu-baseline --no-e2e --no-read-calibration "$@" 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.readline()); r=d['roofline']
print('| %-44s | %9.1f | %7.2f | %6.1f | %.3f |' % (' '.join(sys.argv[1:]) or 'default (dir2, f64, recon 18)', d['value'], d['ms_per_step']*1e3, r['achieved'], r['frac']))" "$@"; }
echo "| configuration | GFLOP/s | us/apply | algorithmic GB/s | frac of measured copy peak |"
echo "|---|---|---|---|---|"
run
run --kernel site
run --kernel dir4
run --precision f32
run --precision mixed
run --recon 12
run --recon 9
run --precision f32 --recon 12
run --precision f32 --recon 9
run --precision mixed --recon 12
run --precision mixed --recon 9
run --nrhs 2
run --nrhs 4
run --nrhs 8
run --precision f32 --nrhs 8
run --nrhs 8 --layout blocked
run --precision f32 --nrhs 8 --layout blocked
run --precision mixed --nrhs 8 --layout blocked
run --precision f32 --nrhs 4 --layout blocked
run --stage
run --local 48,48,48,48
run --local 48,48,48,48 --precision f32
run --local 48,48,48,48 --recon 12
run --force-halo 8
run --force-halo 12
run --force-halo 8 --overlap dirs
