set -x
mkdir -p gpurun_out
timeout 600 python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
for n in 2 4; do
  timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node $n --master-addr 127.0.0.1 --master-port 2951$n \
     bench.py --gpus $n --colocate --steps 50 --warmup 3 > gpurun_out/bench_colocate_$n.json 2> gpurun_out/bench_colocate_$n.err
  echo "rc=$?"; cat gpurun_out/bench_colocate_$n.json; tail -3 gpurun_out/bench_colocate_$n.err
done
timeout 600 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29520 \
   bench.py --impl reference --gpus 2 --steps 20 --warmup 2 > gpurun_out/bench_ref_n2.json 2> gpurun_out/bench_ref_n2.err
echo "rc=$?"; cat gpurun_out/bench_ref_n2.json; tail -3 gpurun_out/bench_ref_n2.err
