# streaming-path iteration: full GPU parity suite, HBM sweep (B <= 8 rows are the streaming path), C2 bench
TAG=${1:-si}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 900 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 1500 python scripts/hbm_sweep.py 100000000 2 > gpurun_out/${TAG}_hbm_sweep.jsonl 2> gpurun_out/${TAG}_hbm_sweep.err
tail -2 gpurun_out/${TAG}_hbm_sweep.err
python -c "
import json
for l in open('gpurun_out/${TAG}_hbm_sweep.jsonl'):
    d = json.loads(l); print(d['B'], round(d['scan_ms'], 3), round(d['table_gbs']), round(d['frac_of_measured_hbm'], 3), d['parity'])"
timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
python -c "import json; d=json.loads(open('gpurun_out/${TAG}_bench.json').read().strip().splitlines()[-1]); print('C2', round(d['value']/1e6,2), 'Mq/s scan', round(d['stages_ms']['scan_ms'],3), d['roofline']['kernel'])"
