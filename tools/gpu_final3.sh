# usage: bash tools/gpu_final3.sh: end-of-session evidence with the final build: smoke, full GPU
# suite, default bench (+ clocks), the ncu launch list of the bench command and ncu --set full of
# the headline kernel
mkdir -p gpurun_out/final3
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1 > gpurun_out/final3/smoke.txt
timeout 2400 python -m pytest tests -m gpu -q --timeout 600 2>&1 | tail -4 > gpurun_out/final3/gpu_tests.txt
timeout 600 python bench.py > gpurun_out/final3/bench.json 2> gpurun_out/final3/bench.err
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/final3/launches.csv python bench.py --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dslash_kernel -s 5 -c 1 -o gpurun_out/final3/prof_headline -f python bench.py --steps 8 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
ncu -i gpurun_out/final3/prof_headline.ncu-rep --page details --csv > gpurun_out/final3/prof_headline_details.csv 2>&1
ncu -i gpurun_out/final3/prof_headline.ncu-rep --page raw --csv > gpurun_out/final3/prof_headline_raw.csv 2>&1
cat gpurun_out/final3/smoke.txt gpurun_out/final3/gpu_tests.txt gpurun_out/final3/bench.json
