# A/B of prebuilt libspg.so variants: SOS="build/a.so build/b.so" CONFIGS="webbase1m ..." bash tools/so_ab.sh
# prints symbolic / numeric ms per variant and config (bench.py, 20 timed steps)
mkdir -p gpurun_out
for so in $SOS; do
  cp $so paper_conf_ipps_ramamoorthybsk15_b200/libspg.so
  for c in ${CONFIGS:-webbase1m}; do
    timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/ab.log 2>&1
    python - "$so" "$c" <<'PY'
import json, sys
try:
    d = json.loads(open("gpurun_out/ab.log").read().strip().splitlines()[-1])
    p = d["phases"]
    print(f"{sys.argv[1]:28s} {sys.argv[2]:11s} value={d['value']:7.2f} sym={p['symbolic_ms']:.3f} num={p['numeric_ms']:.4f}")
except Exception as e:
    print(sys.argv[1], sys.argv[2], "FAILED", open("gpurun_out/ab.log").read()[-500:])
PY
  done
done
