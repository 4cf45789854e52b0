set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 600 python -m pytest tests -m gpu -x -q --timeout 300 -k "c_api_demo" 2>&1 | tail -2
./examples/c_api_demo; ./examples/c_api_demo 16 16 16 16
timeout 300 python bench.py --local 16,16,16,16 --flush-l2 --steps 500 --no-e2e --no-cpu-baseline > gpurun_out/bench_16_flush.json 2> gpurun_out/bench_16_flush.err; cat gpurun_out/bench_16_flush.json
timeout 300 python bench.py --local 16,16,16,16 --steps 500 --no-e2e --no-cpu-baseline > gpurun_out/bench_16_noflush.json 2>&1; python -c "import json; d=json.load(open('gpurun_out/bench_16_noflush.json')); print('16^4 no flush', d['value'], d['roofline']['frac'])"
timeout 600 python bench.py --steps 300 --no-e2e > gpurun_out/bench_cpu1.json 2>/dev/null; python -c "import json; d=json.load(open('gpurun_out/bench_cpu1.json')); print(d['cpu_baseline'])"
