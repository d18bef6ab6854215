# Round-end evidence on one B200: parity tests (rmat23 on every row included), smoke, bench lines
# (every BASELINE config, reference arm), ncu launch lists (webbase1m, citpatents, rmat23) + DRAM
# traffic of the numeric phase, one ncu --set full of k_numeric and of k_tile_rank, the alpha
# sweep, the ablations, compute-sanitizer.  Everything lands in gpurun_out/.
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 1500 python -m pytest tests -q -m gpu -s > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; grep -E "passed|failed|rmat23:" gpurun_out/pytest_gpu.log | tail -3
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke.log
M=gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum
timeout 600 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --profile > gpurun_out/ncu_bench.log 2>&1
python tools/ncu_sum.py gpurun_out/launches.csv > gpurun_out/launches_summary.txt; cat gpurun_out/launches_summary.txt
python tools/traffic.py gpurun_out/launches.csv webbase1m gpurun_out
cp gpurun_out/traffic_webbase1m.json profiles/traffic_webbase1m.json  # the bench line below reads this capture's traffic
timeout 600 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_cit.csv python bench.py --profile --config citpatents --steps 20 > gpurun_out/ncu_cit.log 2>&1
python tools/ncu_sum.py gpurun_out/launches_cit.csv > gpurun_out/launches_citpatents.txt
timeout 900 ncu --metrics $M --clock-control none --csv --log-file gpurun_out/launches_rmat.csv python bench.py --profile --config rmat23 --steps 2 --warmup 3 > gpurun_out/ncu_rmat.log 2>&1
python tools/ncu_sum.py gpurun_out/launches_rmat.csv > gpurun_out/launches_rmat23.txt
timeout 900 python bench.py --out gpurun_out/bench_webbase1m.jsonl > gpurun_out/bench.log 2>&1; tail -1 gpurun_out/bench.log | cut -c1-400
timeout 600 python bench.py --impl reference --steps 3 --warmup 3 --out gpurun_out/bench_reference.jsonl > gpurun_out/bench_ref.log 2>&1; tail -1 gpurun_out/bench_ref.log | cut -c1-300
for c in webgoogle citpatents ab2m cl10k; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --out gpurun_out/bench_configs.jsonl > gpurun_out/bench_$c.log 2>&1; tail -1 gpurun_out/bench_$c.log | cut -c1-200
done
timeout 1200 python bench.py --config rmat23 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --out gpurun_out/bench_rmat23.jsonl > gpurun_out/bench_rmat.log 2>&1; tail -1 gpurun_out/bench_rmat.log | cut -c1-400
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_numeric" -s 3 -c 1 -o gpurun_out/prof_numeric -f python bench.py --profile > gpurun_out/ncu_full.log 2>&1; echo "ncu numeric rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:"k_tile_rank" -s 1 -c 1 -o gpurun_out/prof_tile -f python bench.py --profile > gpurun_out/ncu_tile.log 2>&1; echo "ncu tile rc=$?"
timeout 1800 python tools/alpha_sweep.py --steps 3 --out gpurun_out/r02_alpha_sweep.jsonl > gpurun_out/alpha.log 2>&1; echo "alpha rc=$?"; grep summary gpurun_out/r02_alpha_sweep.jsonl
for c in webbase1m citpatents; do
  timeout 1200 python tools/ablation.py --config $c --out gpurun_out/r02_ablation.jsonl > gpurun_out/ablation_$c.log 2>&1; echo "ablation $c rc=$?"
done
# tools/sanitize.sh: compute-sanitizer is closed on this GPU pool (see profiles/r02_sanitizer.txt)
