# usage: bash tools/gpu_final5_ncu.sh: ncu --set full of the headline stencil launch, current build
mkdir -p gpurun_out/final5
timeout 600 ncu --set full --clock-control none --import-source on -k regex:dslash_kernel -s 5 -c 1 -o gpurun_out/final5/prof_headline -f python bench.py --steps 8 --warmup 3 --no-cpu-baseline --no-e2e > /dev/null 2>&1
echo "ncu rc=$?"
ncu -i gpurun_out/final5/prof_headline.ncu-rep --page details --csv > gpurun_out/final5/prof_headline_details.csv 2>&1
ncu -i gpurun_out/final5/prof_headline.ncu-rep --page raw --csv > gpurun_out/final5/prof_headline_raw.csv 2>&1
