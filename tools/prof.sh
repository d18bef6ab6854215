# build, launch list (ncu timing of every kernel) and ncu --set full of $KERNELS on $CONFIG
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
C=${CONFIG:-webbase1m}
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
if [ "${PYT:-}" = "all" ]; then timeout 1200 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log;
elif [ -n "${PYT:-}" ]; then timeout 900 python -m pytest tests -x -q -m gpu -k "fig2 or random_int or power_law_rows or thresholds or big_tiles or fp32_power or long_rows or rerun or config_full or columns_up" > gpurun_out/pytest_gpu.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/pytest_gpu.log; fi
timeout 300 python bench.py --config $C --steps 10 --warmup 3 --no-cpu-baseline --no-e2e ${BENCH_ARGS:-} > gpurun_out/bench_$C.log 2>&1; tail -1 gpurun_out/bench_$C.log | cut -c1-700
timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/launches_$C.csv python bench.py --profile --config $C ${BENCH_ARGS:-} > gpurun_out/ncu_bench.log 2>&1
python tools/ncu_sum.py gpurun_out/launches_$C.csv
for k in ${KERNELS:-}; do
  timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base demangled -k regex:"$k" -s ${KSKIP:-3} -c 1 -o gpurun_out/prof_${C}_$(echo $k | tr -cd "a-z_0-9") -f \
    python bench.py --profile --config $C ${BENCH_ARGS:-} > gpurun_out/ncu_$k.log 2>&1; echo "$k rc=$?"
done
