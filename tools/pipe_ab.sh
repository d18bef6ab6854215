# numeric software pipeline (SPG_NUM_PIPE): parity with the variant built, then bench A/B
mkdir -p gpurun_out
SPG_NVCC_FLAGS="-DSPG_NUM_PIPE=1 -DSPG_NUM_MINB=4" python -c "from paper_conf_ipps_ramamoorthybsk15_b200 import build as b; b.build(force=True)" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_pipe.log 2>&1; echo "pytest(pipe,minb4) rc=$?"; tail -2 gpurun_out/pytest_pipe.log
FLAGSETS="-DSPG_NUM_PIPE=0|-DSPG_NUM_PIPE=1 -DSPG_NUM_MINB=5|-DSPG_NUM_PIPE=1 -DSPG_NUM_MINB=4|-DSPG_NUM_PIPE=1 -DSPG_NUM_MINB=3|-DSPG_NUM_PIPE=0" bash tools/flag_ab.sh
FLAGSETS="-DSPG_NUM_PIPE=0|-DSPG_NUM_PIPE=1 -DSPG_NUM_MINB=4|-DSPG_NUM_PIPE=1 -DSPG_NUM_MINB=3" BENCH_ARGS="--config citpatents" bash tools/flag_ab.sh
