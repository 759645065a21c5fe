# A/B of scan-kernel variants on the GPU box: GPU parity suite with the candidate forced, then the
# C2 bench per variant.  usage: bash scripts/gpu_ab.sh <tag> <candidate> "<variants to bench>" [bench args]
TAG=${1:-ab}; CAND=${2:-6}; VARS=${3:-"5 6"}; shift 3; EXTRA="$*"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
TM_SCAN_VARIANT=$CAND timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -4
for v in $VARS; do
  TM_SCAN_VARIANT=$v timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline $EXTRA > gpurun_out/${TAG}_v$v.json 2> gpurun_out/${TAG}_v$v.err
  python -c "import json; d=json.loads(open('gpurun_out/${TAG}_v$v.json').read().strip().splitlines()[-1]); print('variant $v', round(d['value']/1e6,2), 'Mq/s scan', round(d['stages_ms']['scan_ms'],3), 'frac', round(d['roofline']['frac'],3), 'tests', d['path_stats']['tile_tests'], 'checks', d['path_stats']['pair_checks'])" || tail -3 gpurun_out/${TAG}_v$v.err
done
