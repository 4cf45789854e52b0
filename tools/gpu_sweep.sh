set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
python tools/sweep.py --dims 32,32,32,32 --steps 400 > gpurun_out/sweep2_32.jsonl 2>&1
python tools/sweep.py --dims 48,48,48,48 --steps 60 --blocks 128,256 > gpurun_out/sweep2_48.jsonl 2>&1
cat gpurun_out/sweep2_*.jsonl
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -5
