# final-state check: parity tests, smoke, headline bench line, other configs
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests -q -m gpu > gpurun_out/pytest_final.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/pytest_final.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.log 2>&1; echo "smoke rc=$?"; tail -1 gpurun_out/smoke_final.log
timeout 600 python bench.py --out gpurun_out/bench_final.jsonl > gpurun_out/bench_final.log 2>&1; tail -1 gpurun_out/bench_final.log | cut -c1-300
for c in webgoogle citpatents ab2m; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --out gpurun_out/bench_final.jsonl > gpurun_out/bench_$c.log 2>&1; tail -1 gpurun_out/bench_$c.log | cut -c1-200
done
timeout 900 python bench.py --config rmat23 --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --out gpurun_out/bench_final.jsonl > gpurun_out/bench_rmat.log 2>&1; tail -1 gpurun_out/bench_rmat.log | cut -c1-200
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --profile > gpurun_out/ncu_bench.log 2>&1
python tools/ncu_sum.py gpurun_out/launches.csv > gpurun_out/launches_summary.txt; cat gpurun_out/launches_summary.txt
