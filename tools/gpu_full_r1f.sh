# usage: bash tools/gpu_full_r1f.sh: smoke, full GPU suite, default bench (after push + recon-9)
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.smoke(); print('smoke ok')" 2>&1 | tail -2
timeout 2400 python -m pytest tests -m gpu -q --timeout 600 2>&1 | tail -8 > gpurun_out/gpu_tests_r1f.txt
cat gpurun_out/gpu_tests_r1f.txt
timeout 600 python bench.py > gpurun_out/bench_r1f.json 2> gpurun_out/bench_r1f.err; cat gpurun_out/bench_r1f.json
echo done
