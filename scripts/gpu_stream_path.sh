# streaming (small-batch) path: parity tests, C2 bench of the first variant, then the HBM sweep per variant
# usage: bash scripts/gpu_stream_path.sh "<variants>"
VARS=${1:-"5 0"}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 900 python -m pytest tests -m gpu -x -q -k "small or c1_single or every_scan or fuzz" 2>&1 | tail -3
V0=${VARS%% *}
TM_SCAN_VARIANT=$V0 timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/stream_c2_v$V0.json 2>&1
python -c "import json; d=json.loads(open('gpurun_out/stream_c2_v$V0.json').read().strip().splitlines()[-1]); print('C2', round(d['value']), 'scan_ms', round(d['roofline']['kernel_ms'],3))"
for v in $VARS; do
  TM_SCAN_VARIANT=$v timeout 900 python scripts/hbm_sweep.py 100000000 2 > gpurun_out/hbm_sweep_v$v.jsonl 2> gpurun_out/hbm_sweep_v$v.err
  echo "variant $v"; python -c "
import json
for l in open('gpurun_out/hbm_sweep_v$v.jsonl'):
    d = json.loads(l); print(d['B'], round(d['scan_ms'], 3), round(d['table_gbs']), round(d['frac_of_measured_hbm'], 3), d['parity'])"
done
