# k_numeric grid: resident grid-stride (-DSPG_NUM_RESIDENT_GRID) vs one block per chunk (default; -DSPG_NUM_FULLGRID is a no-op tag)
mkdir -p gpurun_out
for c in webbase1m webgoogle citpatents; do
  FLAGSETS="-DSPG_NUM_RESIDENT_GRID|-DSPG_NUM_FULLGRID|-DSPG_NUM_RESIDENT_GRID|-DSPG_NUM_FULLGRID" BENCH_ARGS="--config $c" bash tools/flag_ab.sh
done
SPG_NVCC_FLAGS="-DSPG_NUM_FULLGRID" python -c "from paper_conf_ipps_ramamoorthybsk15_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_grid.log 2>&1; echo "pytest(fullgrid) rc=$?"; tail -1 gpurun_out/pytest_grid.log
