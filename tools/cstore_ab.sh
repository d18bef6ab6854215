# C store policy in k_numeric (SPG_C_STORE): bench A/B on three configs
mkdir -p gpurun_out
for c in webbase1m webgoogle citpatents; do
  FLAGSETS="-DSPG_C_STORE=0|-DSPG_C_STORE=1|-DSPG_C_STORE=0|-DSPG_C_STORE=1" BENCH_ARGS="--config $c" bash tools/flag_ab.sh
done
SPG_NVCC_FLAGS="-DSPG_C_STORE=1" python -c "from paper_conf_ipps_ramamoorthybsk15_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
timeout 600 python -m pytest tests -x -q -m gpu -k numeric > gpurun_out/pytest_cstore.log 2>&1; echo "pytest(cstore=1) rc=$?"; tail -1 gpurun_out/pytest_cstore.log
