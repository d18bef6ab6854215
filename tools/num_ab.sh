# A/B of numeric-kernel options: launch-list times of the numeric kernels per setting
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || tail gpurun_out/build.log
i=0
for v in ${VARIANTS:-"SPG_PACK_B=0" "SPG_PACK_B=1"}; do
  i=$((i+1))
  echo "== $v"
  env $v timeout 300 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/ab_$i.csv python bench.py --profile > gpurun_out/ab_$i.log 2>&1 || tail -5 gpurun_out/ab_$i.log
  python tools/ncu_sum.py gpurun_out/ab_$i.csv | grep -v "scan\|k_tiles\|classify\|Fill"
done
