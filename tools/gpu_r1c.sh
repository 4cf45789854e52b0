# usage: bash tools/gpu_r1c.sh  (GPU box, repo root): NCCL self-exchange tests + bench, HBM/PCIe ceilings
set -x
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 900 python -m pytest tests -m gpu -q --timeout 400 -k "nccl or cg_self_halo" 2>&1 | tail -8 > gpurun_out/gpu_tests_r1c.txt
cat gpurun_out/gpu_tests_r1c.txt
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/stream_peak tools/stream_peak.cu && timeout 300 /tmp/stream_peak > gpurun_out/stream_peak.txt 2>&1
cat gpurun_out/stream_peak.txt
timeout 300 python tools/pcie_peak.py > gpurun_out/pcie_peak.json 2>&1; cat gpurun_out/pcie_peak.json
run() { name=$1; shift; timeout 300 python bench.py --steps 1000 --no-cpu-baseline "$@" > gpurun_out/bench_$name.json 2> gpurun_out/bench_$name.err; python -c "
import json,sys; d=json.load(open('gpurun_out/bench_$name.json')); r=d['roofline']
print('$name', d['value'], d['unit'], 'frac', r['frac'], 'us', r['avg_launch_us'], d['ms_per_step'], 'e2e', (d.get('e2e') or {}).get('value'))" || tail -5 gpurun_out/bench_$name.err; }
run selfnccl_t --force-halo 8 --self-nccl --local 32,32,32,32
run selfnccl_tz --force-halo 12 --self-nccl --local 32,32,32,32
run selfcopy_t --force-halo 8 --local 32,32,32,32
NCCL_DEBUG=INFO timeout 120 python bench.py --steps 50 --warmup 3 --no-cpu-baseline --no-e2e --force-halo 8 --self-nccl 2>&1 | grep -i "nccl.*\(version\|channel\|P2P\|SHM\)" | head -20 > gpurun_out/nccl_self_info.txt
echo done
