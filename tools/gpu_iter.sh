# build, parity tests, bench, launch list, then ncu --set full of $KERNELS (regex each)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 python -m pytest tests -x -q -m gpu ${PYTEST_ARGS:-} > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"
tail -4 gpurun_out/pytest_gpu.log
timeout 600 python bench.py --steps 30 --warmup 5 --no-cpu-baseline ${BENCH_ARGS:-} > gpurun_out/bench.log 2>&1; tail -1 gpurun_out/bench.log | cut -c1-1800
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/launches.csv python bench.py --profile ${BENCH_ARGS:-} > gpurun_out/ncu_bench.log 2>&1
python tools/ncu_sum.py gpurun_out/launches.csv
for k in ${KERNELS:-}; do
  timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"$k" -s ${KSKIP:-3} -c 1 -o gpurun_out/prof_$(echo $k | tr -cd "a-z_0-9") -f \
    python bench.py --profile ${BENCH_ARGS:-} > gpurun_out/ncu_$k.log 2>&1; echo "$k rc=$?"
done
