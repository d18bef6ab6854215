# per-path symbolic timing for each .so and config
for so in $SOS; do
  cp $so paper_conf_ipps_ramamoorthybsk15_b200/libspg.so
  for c in ${CONFIGS}; do
    timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cpu-baseline --no-e2e $EXTRA > gpurun_out/ab.log 2>&1
    tail -1 gpurun_out/ab.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['phases']; print('$so $c', round(d['value'],2), round(p['symbolic_ms'],3), round(p['numeric_ms'],3), p['symbolic_path_ms'])" || tail -3 gpurun_out/ab.log
  done
done
