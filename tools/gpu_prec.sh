set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
for p in f32 mixed; do
  python bench.py --precision $p --steps 1000 --no-cpu-baseline > gpurun_out/bench_$p.json 2> gpurun_out/bench_$p.err
  cat gpurun_out/bench_$p.json; tail -2 gpurun_out/bench_$p.err
done
python tools/sweep.py --dims 32,32,32,32 --steps 300 --blocks 64,128 --minb 2,3 --kernels site,dir2,dir4 --precision f32 > gpurun_out/sweep_f32.jsonl 2>&1
cat gpurun_out/sweep_f32.jsonl
