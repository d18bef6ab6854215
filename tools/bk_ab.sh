# A/B of the light-tile bucket size (SPG_TILE_BK): bench line + phase split per setting
for bk in ${BKS:-4 2 3}; do
  SPG_NVCC_FLAGS="-DSPG_TILE_BK=$bk" python -c "from paper_conf_ipps_ramamoorthybsk15_b200 import build as b; b.build(force=True)" > /dev/null 2>&1 || echo "build fail $bk"
  timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/bk.log 2>&1
  tail -1 gpurun_out/bk.log | python -c "import json,sys; d=json.loads(sys.stdin.read()); print('BK=$bk', round(d['value'],2), round(d['phases']['symbolic_ms'],3), d['phases']['symbolic_path_ms'])"
  SPG_NVCC_FLAGS="-DSPG_TILE_BK=$bk -DSPG_PHASE_PROF" python -c "from paper_conf_ipps_ramamoorthybsk15_b200 import build as b; b.build(force=True)" > /dev/null 2>&1
  python tools/phase_prof.py webbase1m | tr '\n' ' '; echo
done
