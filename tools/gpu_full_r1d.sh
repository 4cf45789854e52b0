# usage: bash tools/gpu_full_r1d.sh: full GPU suite + smoke + default bench + ncu --set full of the 4/8-RHS kernels
set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 2400 python -m pytest tests -m gpu -q --timeout 600 2>&1 | tail -6 > gpurun_out/gpu_tests_r1d.txt
cat gpurun_out/gpu_tests_r1d.txt
timeout 600 python bench.py > gpurun_out/bench_r1d.json 2> gpurun_out/bench_r1d.err; cat gpurun_out/bench_r1d.json
for n in 4 8; do
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dslash_kernel -s 5 -c 1 -o gpurun_out/prof_n$n -f python bench.py --steps 8 --warmup 3 --no-cpu-baseline --no-e2e --kernel site --nrhs $n > /dev/null 2>&1
ncu -i gpurun_out/prof_n$n.ncu-rep --page details --csv > gpurun_out/prof_n${n}_details.csv 2>&1
done
echo done
