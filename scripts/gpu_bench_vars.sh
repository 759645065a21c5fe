# C2 bench per forced scan variant (no parity suite).  usage: bash scripts/gpu_bench_vars.sh <tag> "<variants>" [bench args]
TAG=${1:-bv}; VARS=${2:-"5"}; shift 2; EXTRA="$*"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
for v in $VARS; do
  TM_SCAN_VARIANT=$v timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline $EXTRA > gpurun_out/${TAG}_v$v.json 2> gpurun_out/${TAG}_v$v.err
  python -c "import json; d=json.loads(open('gpurun_out/${TAG}_v$v.json').read().strip().splitlines()[-1]); print('variant $v', d['config']['workload'], round(d['value']/1e6,3), 'Mq/s scan', round(d['stages_ms']['scan_ms'],3), 'frac', round(d['roofline']['frac'],3))" || tail -3 gpurun_out/${TAG}_v$v.err
done
