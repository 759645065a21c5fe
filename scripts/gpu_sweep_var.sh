# HBM sweep per forced variant (auto = the library's choice) + C2 bench.  usage: bash scripts/gpu_sweep_var.sh <tag> "<auto 5 0 ...>"
TAG=${1:-sv}; VARS=${2:-"auto 5"}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for V in $VARS; do
  if [ $V = auto ]; then unset TM_SCAN_VARIANT; else export TM_SCAN_VARIANT=$V; fi
  timeout 1500 python scripts/hbm_sweep.py 100000000 2 > gpurun_out/${TAG}_hbm_$V.jsonl 2> gpurun_out/${TAG}_hbm_$V.err
  tail -2 gpurun_out/${TAG}_hbm_$V.err
  python -c "
import json
for l in open('gpurun_out/${TAG}_hbm_$V.jsonl'):
    d = json.loads(l); print('$V', d['B'], d['variant'], round(d['scan_ms'], 3), round(d['table_gbs']), round(d['frac_of_measured_hbm'], 3), d['parity'], d['work_items'])"
done
unset TM_SCAN_VARIANT
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
python -c "import json; d=json.loads(open('gpurun_out/${TAG}_bench.json').read().strip().splitlines()[-1]); print('C2', round(d['value']/1e6,2), 'Mq/s scan', round(d['stages_ms']['scan_ms'],3), d['roofline']['kernel'])"
