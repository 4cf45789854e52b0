# CG per-iteration time with the double-double reductions, and multi-RHS block sizes
for i in 1 2; do timeout 300 python tools/bench_cg.py; done
timeout 300 python tools/bench_cg.py --solver mixed-cg
timeout 300 python tools/bench_cg.py --force-halo 8 --transport p2p --push
run() { timeout 300 python bench.py --steps 300 --warmup 10 --no-cpu-baseline --no-e2e --no-read-calibration "$@" 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.readline()); r=d['roofline']; print('$*', d['value'], r['frac'], r['avg_launch_us'])"; }
for n in 2 4; do for b in 64 128 256; do run --nrhs $n --block $b; done; done
run --nrhs 8
run --nrhs 8 --precision f32
run --nrhs 8 --precision f32 --block 64
