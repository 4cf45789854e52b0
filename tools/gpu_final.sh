# final refresh: smoke, full GPU suite, default bench (+cpu baseline), reference arm, ncu launch list + full capture
set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -3
timeout 2400 python -m pytest tests -m gpu -q --timeout 400 2>&1 | tail -6
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > gpurun_out/clocks_final.csv &
SMI=$!
timeout 600 python bench.py > gpurun_out/bench_final.json 2> gpurun_out/bench_final.err
kill $SMI
cat gpurun_out/bench_final.json; tail -2 gpurun_out/bench_final.err
timeout 900 python bench.py --impl reference --steps 100 --warmup 3 > gpurun_out/bench_final_ref.json 2> gpurun_out/bench_final_ref.err
cat gpurun_out/bench_final_ref.json
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_final.csv \
    python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:dslash_kernel -s 5 -c 2 \
    -o gpurun_out/prof_final -f python bench.py --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_final.log 2>&1
tail -1 gpurun_out/ncu_final.log
