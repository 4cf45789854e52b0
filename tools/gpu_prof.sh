# ncu launch list + full capture of both kernel variants (run on the GPU box from the repo root)
set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build()"
python tools/sweep.py --dims 32,32,32,32 > gpurun_out/sweep_32.jsonl 2>&1
python tools/sweep.py --dims 16,16,16,16 --blocks 64,128,256 > gpurun_out/sweep_16.jsonl 2>&1
python tools/sweep.py --dims 48,48,48,48 --blocks 128,256 --steps 100 > gpurun_out/sweep_48.jsonl 2>&1
cat gpurun_out/sweep_*.jsonl
ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_site.csv \
    python bench.py --kernel site --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
for k in site dir4; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:dslash_${k}_kernel -s 5 -c 2 \
    -o gpurun_out/prof_$k -f python bench.py --kernel $k --steps 10 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ncu_$k.log 2>&1
  tail -3 gpurun_out/ncu_$k.log
done
ls -la gpurun_out
