# heavy-row column-span tiles (SPG_BMP_SPAN): parity with the default build, then bench A/B
mkdir -p gpurun_out
python -c "from paper_conf_ipps_ramamoorthybsk15_b200 import build as b; b.build(force=True)" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_span.log 2>&1; echo "pytest(span) rc=$?"; tail -2 gpurun_out/pytest_span.log
for c in webbase1m citpatents webgoogle ab2m; do
  FLAGSETS="-DSPG_BMP_SPAN=0|-DSPG_BMP_SPAN=1|-DSPG_BMP_SPAN=0|-DSPG_BMP_SPAN=1" BENCH_ARGS="--config $c" bash tools/flag_ab.sh
done
FLAGSETS="-DSPG_BMP_SPAN=0|-DSPG_BMP_SPAN=1" BENCH_ARGS="--config rmat23 --steps 3 --warmup 3" bash tools/flag_ab.sh
