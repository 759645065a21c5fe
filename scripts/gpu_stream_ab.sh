# HBM sweep with the library's own variant choice and with variant 0 forced (direct streaming check at
# every B <= 8), plus GPU parity suite.  usage: bash scripts/gpu_stream_ab.sh <tag>
TAG=${1:-sab}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -2
for V in auto 0; do
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
