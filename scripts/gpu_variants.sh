# compare scan-kernel variants (TM_SCAN_VARIANT) on correctness + C2 bench (+ optional config)
# usage: bash scripts/gpu_variants.sh "<variants>" [config]
VARS=${1:-"0 1 2 3"}; CFG=${2:-C2}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
for v in $VARS; do
  echo "=== variant $v"
  TM_SCAN_VARIANT=$v timeout 900 python -m pytest tests -m gpu -x -q -k "c1_single or edge or c2_full or overflow" 2>&1 | tail -2
  TM_SCAN_VARIANT=$v timeout 900 python bench.py --config $CFG --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/var_${CFG}_$v.json 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/var_${CFG}_$v.json').read().strip().splitlines()[-1]); print(round(d['value']), 'scan_ms', round(d['roofline']['kernel_ms'],3), 'frac', round(d['roofline']['frac'],3))"
done
