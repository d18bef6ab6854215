# one ncu --set full capture per kernel regex given in $KERNELS (space separated), 1 launch each
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
for k in ${KERNELS}; do
  timeout 900 ncu --set full --clock-control none --import-source on -k regex:"$k" -s 3 -c 1 -o gpurun_out/prof_$k -f \
    python bench.py --profile ${BENCH_ARGS:-} > gpurun_out/ncu_$k.log 2>&1; echo "$k rc=$?"
done
