set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
python tools/probe_overlap.py 48,48,48,6 8
python tools/probe_overlap.py 32,32,32,32 8
timeout 300 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/ncu_dirs_t8.csv python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --local 48,48,48,6 --force-halo 8 --overlap dirs > /dev/null 2>&1
grep -o '"[a-zA-Z_:<>, 0-9]*dslash[^"]*","[^"]*","[^"]*","gpu__time_duration.sum","[^"]*","[0-9.]*"' gpurun_out/ncu_dirs_t8.csv | tail -12
tail -12 gpurun_out/ncu_dirs_t8.csv | cut -c1-300
