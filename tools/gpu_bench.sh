# full bench (default config) + ncu launch list + ncu --set full of the default kernel
set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > gpurun_out/clocks.csv &
SMI=$!
python bench.py > gpurun_out/bench_default.json 2> gpurun_out/bench_default.err
kill $SMI
cat gpurun_out/bench_default.json; tail -3 gpurun_out/bench_default.err
python bench.py --impl reference --steps 50 --warmup 3 > gpurun_out/bench_reference.json 2> gpurun_out/bench_reference.err
cat gpurun_out/bench_reference.json; tail -3 gpurun_out/bench_reference.err
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_default.csv \
    python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dslash_kernel -s 5 -c 2 \
    -o gpurun_out/prof_dir2 -f python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_dir2.log 2>&1
tail -2 gpurun_out/ncu_dir2.log
