# GPU parity suite + C3 bench line.  usage: bash scripts/gpu_c3.sh <tag>
TAG=${1:-c3}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3
timeout 1800 python bench.py --config C3 --steps 5 --warmup 3 --cpu-s 20 > gpurun_out/${TAG}_C3_bench.json 2> gpurun_out/${TAG}_C3_bench.err
tail -1 gpurun_out/${TAG}_C3_bench.err; python -c "import json; d=json.loads(open('gpurun_out/${TAG}_C3_bench.json').read().strip().splitlines()[-1]); print('C3', d['value'], d['e2e']['value'], d['stages_ms'], d['roofline']['frac'], d['roofline']['kernel'], d['cpu_baseline']['value'])"
