# A/B of runtime env options: ENVSETS="A=1 B=0|A=0" (| separated); bench line per variant
IFS='|' read -ra SETS <<< "${ENVSETS}"
for es in "${SETS[@]}"; do
  env $es timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e ${BENCH_ARGS:-} > gpurun_out/envab.log 2>&1
  tail -1 gpurun_out/envab.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$es]', round(d['value'],2), round(d['phases']['symbolic_ms'],3), round(d['phases']['numeric_ms'],3))" || tail -3 gpurun_out/envab.log
done
