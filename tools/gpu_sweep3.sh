set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 900 python tools/sweep.py --dims 32,32,32,32 --steps 1000 --kernels site,dir2,dir4 --blocks 64,96,128,256 --minb 2,3,4 > gpurun_out/sweep3_32.jsonl 2>&1
sort -t: -k6 gpurun_out/sweep3_32.jsonl | python -c "
import sys,json
rows=[json.loads(l) for l in open('gpurun_out/sweep3_32.jsonl') if l.startswith('{')]
rows.sort(key=lambda r: r['us_per_apply'])
for r in rows[:12]: print(r['kernel'], r['block'], r['minb'], r['us_per_apply'], r['algo_gbs'], r['gflops'])
"
timeout 900 python tools/sweep.py --dims 48,48,48,48 --steps 200 --kernels site,dir2 --blocks 64,128 --minb 2,3 > gpurun_out/sweep3_48.jsonl 2>&1
cat gpurun_out/sweep3_48.jsonl
