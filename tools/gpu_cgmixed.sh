# usage: bash tools/gpu_cgmixed.sh: mixed-precision CG tests + solve-time benchmarks at 32^4
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests/test_gpu_solver.py -q --timeout 400 2>&1 | tail -5
for args in "--solver cg" "--solver cg --precision mixed" "--solver mixed-cg --inner-tol 1e-4" "--solver mixed-cg --inner-tol 1e-3" "--solver mixed-cg --inner-tol 1e-2" "--solver mixed-cg --inner-tol 1e-5"; do
  timeout 300 python tools/bench_cg.py $args 2>/dev/null | tee -a gpurun_out/bench_cgmixed.jsonl
done
echo done
