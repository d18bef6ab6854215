# persisting-L2 window over B during numeric (SPG_L2_PERSIST), with and without packed B
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
SPG_L2_PERSIST=1 timeout 600 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_l2p.log 2>&1; echo "pytest(l2p) rc=$?"; tail -1 gpurun_out/pytest_l2p.log
for c in webbase1m citpatents webgoogle; do
  echo "== $c"
  ENVSETS="SPG_L2_PERSIST=0|SPG_L2_PERSIST=1|SPG_L2_PERSIST=2|SPG_PACK_B=1|SPG_PACK_B=1 SPG_L2_PERSIST=1|SPG_PACK_B=1 SPG_L2_PERSIST=2|SPG_L2_PERSIST=0" BENCH_ARGS="--config $c" bash tools/env_ab.sh
done
