# numeric-phase time only for prebuilt .so variants (results may be wrong for probe builds)
for so in $SOS; do
  cp $so paper_conf_ipps_ramamoorthybsk15_b200/libspg.so
  for c in ${CONFIGS:-webbase1m}; do
    timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ab.log 2>&1
    tail -1 gpurun_out/ab.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); p=d['phases']; print('$so $c num', round(p['numeric_ms'],4), 'min', round(p['numeric_ms_min'],4))" || tail -3 gpurun_out/ab.log
  done
done
