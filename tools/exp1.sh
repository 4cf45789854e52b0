set -x
mkdir -p gpurun_out/exp1
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/exp1/build.txt 2>&1
for b in 64 128 256; do
  timeout 300 python bench.py --steps 300 --warmup 10 --no-cpu-baseline --no-e2e --no-read-calibration --kernel site --nrhs 8 --block $b > gpurun_out/exp1/n8_b$b.json 2>gpurun_out/exp1/n8_b$b.err
done
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dslash_kernel -s 3 -c 1 -o gpurun_out/exp1/n8_site python bench.py --kernel site --nrhs 8 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-read-calibration > gpurun_out/exp1/ncu_n8.txt 2>&1
timeout 600 ncu --set full --clock-control none -k regex:dslash_kernel -s 3 -c 1 -o gpurun_out/exp1/n1_dir2 python bench.py --steps 3 --warmup 3 --no-cpu-baseline --no-e2e --no-read-calibration > gpurun_out/exp1/ncu_n1.txt 2>&1
echo done
