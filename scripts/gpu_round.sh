# one full check-in run: smoke + all GPU tests + C2 bench + pinned-variant ncu, then the HBM sweep
# usage: bash scripts/gpu_round.sh <tag>
TAG=${1:-r}
bash scripts/gpu_iter.sh $TAG
timeout 900 python scripts/hbm_sweep.py 100000000 2 > gpurun_out/${TAG}_hbm_sweep.jsonl 2> gpurun_out/${TAG}_hbm_sweep.err
python -c "
import json
for l in open('gpurun_out/${TAG}_hbm_sweep.jsonl'):
    d = json.loads(l); print(d['B'], round(d['scan_ms'], 3), round(d['table_gbs']), round(d['frac_of_measured_hbm'], 3), d['parity'])"
