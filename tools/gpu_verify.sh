# usage: bash tools/gpu_verify.sh TAG  (GPU box, repo root): smoke, GPU tests, default bench, reference arm
TAG=${1:-verify}
set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -3
timeout 2400 python -m pytest tests -m gpu -q --timeout 400 2>&1 | tail -8 > gpurun_out/gpu_tests_$TAG.txt
cat gpurun_out/gpu_tests_$TAG.txt
nvidia-smi --query-gpu=index,clocks.sm,clocks.max.sm,power.draw,clocks_event_reasons.active --format=csv -lms 200 > gpurun_out/clocks_$TAG.csv &
SMI=$!
timeout 600 python bench.py > gpurun_out/bench_$TAG.json 2> gpurun_out/bench_$TAG.err
kill $SMI
cat gpurun_out/bench_$TAG.json; tail -2 gpurun_out/bench_$TAG.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 > gpurun_out/bench_ref_$TAG.json 2> gpurun_out/bench_ref_$TAG.err
cat gpurun_out/bench_ref_$TAG.json
echo done
