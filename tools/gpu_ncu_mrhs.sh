set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 600 ncu --set full --clock-control none -k regex:dslash_kernel -s 3 -c 1 -o gpurun_out/prof_n8 -f \
    python bench.py --kernel site --nrhs 8 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_n8.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:dslash_kernel -s 3 -c 1 -o gpurun_out/prof_n4 -f \
    python bench.py --kernel site --nrhs 4 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_n4.log 2>&1
timeout 600 ncu --set full --clock-control none -k regex:dslash_kernel -s 3 -c 1 -o gpurun_out/prof_f32 -f \
    python bench.py --precision f32 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_f32.log 2>&1
tail -1 gpurun_out/ncu_n8.log gpurun_out/ncu_n4.log gpurun_out/ncu_f32.log
