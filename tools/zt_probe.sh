run() { timeout 300 python bench.py --steps 500 --warmup 20 --no-cpu-baseline --no-e2e --no-read-calibration "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); r=d['roofline']; print('$*', d['value'], r['frac'], r['avg_launch_us'])"; }
run; run --nrhs 8; run --nrhs 4; run --nrhs 2; run --precision f32; run --nrhs 8 --precision f32; run --kernel site; run --recon 9; run --precision mixed
timeout 300 ncu --set full --clock-control none -k regex:dslash -s 5 -c 1 -o gpurun_out/r02_zt/n8 -f python bench.py --nrhs 8 --steps 8 --warmup 3 --no-cpu-baseline --no-e2e --no-read-calibration > /dev/null 2>&1
ncu -i gpurun_out/r02_zt/n8.ncu-rep --page raw --csv > gpurun_out/r02_zt/n8_raw.csv 2>&1
