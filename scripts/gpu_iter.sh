# one iteration on the GPU box: parity tests, bench lines, ncu launch list + full capture of k_scan
# usage: bash scripts/gpu_iter.sh <tag> [pytest -k expr] [extra bench variants "args|args"]
TAG=${1:-iter}
K=${2:-}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
if [ "$K" != "none" ]; then
  if [ -n "$K" ]; then timeout 1500 python -m pytest tests -m gpu -x -q -k "$K" 2>&1 | tail -15;
  else timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -15; fi
fi
timeout 600 python bench.py --steps 10 --warmup 3 --cpu-s 5 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
tail -2 gpurun_out/${TAG}_bench.err; cat gpurun_out/${TAG}_bench.json
IFS='|' read -ra VARS <<< "${3:-}"
i=0
for v in "${VARS[@]}"; do
  i=$((i+1))
  timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline $v > gpurun_out/${TAG}_var$i.json 2>&1
  echo "variant $v:"; python -c "import json,sys; d=json.loads(open('gpurun_out/${TAG}_var$i.json').read().strip().splitlines()[-1]); print(d['value'], d['stages_ms'], d['path_stats'])"
done
# profile the variant the bench's handle tuned to (under ncu the tuner's timings are not meaningful)
VAR=$(python -c "import json,re; d=json.loads(open('gpurun_out/${TAG}_bench.json').read().strip().splitlines()[-1]); print(re.findall(r'variant (\d+)', d['roofline']['kernel'])[0])" 2>/dev/null)
TM_SCAN_VARIANT=${VAR:-5} bash scripts/gpu_profile.sh ${TAG} > gpurun_out/${TAG}_profile.log 2>&1
