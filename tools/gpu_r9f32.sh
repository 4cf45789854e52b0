# usage: bash tools/gpu_r9f32.sh: fp32 / mixed throughput by long-link storage (recon 18 / 12 / 9), 32^4
for prec in f32 mixed; do for r in 18 12 9; do for k in dir2 site; do
timeout 200 python bench.py --precision $prec --recon $r --kernel $k --steps 1000 --warmup 10 --no-cpu-baseline --no-e2e --no-read-calibration 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); print('$prec recon $r $k |', round(d['ms_per_step']*1e3,1), 'us', d['value'], 'GFLOP/s', d['roofline']['frac'], d['roofline']['bytes_per_site'])"
done; done; done
