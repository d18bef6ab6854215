mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1 || { tail -30 gpurun_out/build.log; exit 1; }
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,smsp__inst_executed.sum --clock-control none --csv --log-file gpurun_out/launches_rmat.csv python bench.py --profile --config rmat23 > gpurun_out/ncu_rmat.log 2>&1
python tools/ncu_sum.py gpurun_out/launches_rmat.csv
