# (light_max, tile) grid on the given configs: CONFIGS="webbase1m ..." bash tools/sweep_quick.sh
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
for c in ${CONFIGS:-webbase1m citpatents}; do
for o in ${GRID:-"light_max_flops=1024,tile_flops=3072" "light_max_flops=2048,tile_flops=2048" "light_max_flops=3072,tile_flops=1024" "light_max_flops=2048,tile_flops=3072" "light_max_flops=4096,tile_flops=2048" "light_max_flops=1536,tile_flops=2048" "light_max_flops=2560,tile_flops=1536"}; do
  args=""; for kv in ${o//,/ }; do args="$args --opt $kv"; done
  timeout 200 python bench.py --config $c --steps 10 --warmup 3 --no-cpu-baseline --no-e2e $args > /tmp/o.log 2>&1
  python -c "
import json,sys; d=json.loads(open('/tmp/o.log').read().strip().splitlines()[-1]); p=d['phases']
print('$c', '$o', round(d['value'],2), 'sym', round(p['symbolic_ms'],3), 'num', round(p['numeric_ms'],3), p['symbolic_path_ms'])" || tail -2 /tmp/o.log
done; done
