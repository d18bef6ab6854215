# rmat23 with two threshold settings, and the N=2 path (virtual ranks on one GPU)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for o in "--opt tile_flops=2048 --opt light_max_flops=2048" "--opt tile_flops=1024 --opt light_max_flops=3072"; do
  timeout 900 python bench.py --config rmat23 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e $o > gpurun_out/rmat_opt.log 2>&1
  tail -1 gpurun_out/rmat_opt.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('$o', round(d['value'],2), d['phases']['symbolic_ms'], d['phases']['numeric_ms'], d['phases']['symbolic_path_ms'], d['roofline']['frac'])"
done
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 --master-port 29533 bench.py --gpus 2 --steps 10 --warmup 3 --sim-ranks-on-one-gpu --no-cpu-baseline --no-e2e > gpurun_out/sim2.log 2>&1; echo "sim2 rc=$?"; tail -1 gpurun_out/sim2.log | cut -c1-700
