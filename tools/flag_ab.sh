# A/B of compile-time variants: FLAGSETS="-DX=1|-DX=2" (| separated); bench line per variant
IFS='|' read -ra SETS <<< "${FLAGSETS}"
for fl in "${SETS[@]}"; do
  SPG_NVCC_FLAGS="$fl" python -c "from paper_conf_ipps_ramamoorthybsk15_b200 import build as b; b.build(force=True)" > /dev/null 2>&1 || echo "build fail $fl"
  timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e ${BENCH_ARGS:-} > gpurun_out/flag.log 2>&1
  tail -1 gpurun_out/flag.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('[$fl]', round(d['value'],2), round(d['phases']['symbolic_ms'],3), round(d['phases']['numeric_ms'],3), d['phases']['symbolic_path_ms'])"
done
