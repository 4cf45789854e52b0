set -x
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 300 python -m pytest tests/test_gpu_overlap_fused.py -q -k dryrun 2>&1 | tail -2
python tools/probe_overlap.py 32,32,32,32 8
python tools/probe_overlap.py 48,48,48,6 8
echo done
