# Round-end evidence on one B200: parity tests, smoke, bench lines (every BASELINE config, reference
# arm), ncu launch list + DRAM traffic of the numeric phase, one ncu --set full of k_numeric and
# of k_tile_rank, the alpha sweep and ablations, compute-sanitizer.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -q -m gpu -s > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; grep -E "passed|failed|rmat23:" gpurun_out/pytest_gpu.log | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --profile > gpurun_out/ncu_bench.log 2>&1
python tools/ncu_sum.py gpurun_out/launches.csv > gpurun_out/launches_summary.txt; cat gpurun_out/launches_summary.txt
python tools/traffic.py gpurun_out/launches.csv webbase1m gpurun_out
timeout 900 python bench.py --out gpurun_out/bench_webbase1m.jsonl > gpurun_out/bench.log 2>&1; tail -1 gpurun_out/bench.log | cut -c1-400
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 --out gpurun_out/bench_reference.jsonl > gpurun_out/bench_ref.log 2>&1; tail -1 gpurun_out/bench_ref.log | cut -c1-300
for c in webgoogle citpatents ab2m cl10k; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --out gpurun_out/bench_configs.jsonl > gpurun_out/bench_$c.log 2>&1; tail -1 gpurun_out/bench_$c.log | cut -c1-200
done
timeout 1200 python bench.py --config rmat23 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --out gpurun_out/bench_rmat23.jsonl > gpurun_out/bench_rmat.log 2>&1; tail -1 gpurun_out/bench_rmat.log | cut -c1-400
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_numeric" -s 3 -c 1 -o gpurun_out/prof_numeric -f python bench.py --profile > gpurun_out/ncu_full.log 2>&1; echo "ncu numeric rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_tile_rank" -s 1 -c 1 -o gpurun_out/prof_tile -f python bench.py --profile > gpurun_out/ncu_tile.log 2>&1; echo "ncu tile rc=$?"
timeout 1800 python tools/alpha_sweep.py --steps 3 --out gpurun_out/r02_alpha_sweep.jsonl > gpurun_out/alpha.log 2>&1; echo "alpha rc=$?"; grep summary gpurun_out/r02_alpha_sweep.jsonl
bash tools/sanitize.sh
