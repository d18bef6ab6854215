# A/B of library options on one build: OPTS="none heavy_dual=1" CONFIGS="webbase1m ab2m" bash tools/opt_ab2.sh
mkdir -p gpurun_out
for rep in 1 2; do
for o in $OPTS; do
  for c in ${CONFIGS:-webbase1m}; do
    a=""; [ "$o" != "none" ] && a="--opt $o"
    timeout 300 python bench.py --config $c --steps ${STEPS:-20} --warmup 3 --no-cpu-baseline --no-e2e $a > gpurun_out/ab.log 2>&1
    python - "$o" "$c" <<'PY'
import json, sys
try:
    d = json.loads(open("gpurun_out/ab.log").read().strip().splitlines()[-1])
    p = d["phases"]
    print(f"{sys.argv[1]:28s} {sys.argv[2]:11s} value={d['value']:7.2f} sym={p['symbolic_ms']:.3f} num={p['numeric_ms']:.4f} heavy={p['symbolic_path_ms']['heavy']:.3f} light={p['symbolic_path_ms']['light']:.3f}")
except Exception as e:
    print(sys.argv[1], sys.argv[2], "FAILED", open("gpurun_out/ab.log").read()[-500:])
PY
  done
done
done
