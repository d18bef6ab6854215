# A/B of runtime options: OPTSETS="--opt a=1|--opt a=2" (| separated); bench line per setting
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
IFS='|' read -ra SETS <<< "${OPTSETS}"
for o in "${SETS[@]}"; do
  timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e ${BENCH_ARGS:-} $o > gpurun_out/opt.log 2>&1
  tail -1 gpurun_out/opt.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$o]', round(d['value'],2), round(d['phases']['symbolic_ms'],3), round(d['phases']['numeric_ms'],3), d['phases']['symbolic_path_ms'])"
done
