# full-size lines: C3 + C4 bench (with CPU baseline), C4 sampled parity, C5 sweep.  usage: bash scripts/gpu_big2.sh <tag>
TAG=${1:-big}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 1800 python bench.py --config C3 --steps 5 --warmup 3 --cpu-s 20 > gpurun_out/${TAG}_C3_bench.json 2> gpurun_out/${TAG}_C3_bench.err
tail -1 gpurun_out/${TAG}_C3_bench.err; python -c "import json; d=json.loads(open('gpurun_out/${TAG}_C3_bench.json').read().strip().splitlines()[-1]); print('C3', d['value'], d['e2e']['value'], d['stages_ms'], d['roofline']['frac'], d['roofline']['kernel'], d['cpu_baseline']['value'])"
TM_FULL_SIZE=C4 timeout 2400 python -m pytest tests/test_gpu_full.py -m gpu -x -q -s 2>&1 | tail -6
timeout 2400 python bench.py --config C4 --steps 3 --warmup 3 --cpu-s 20 > gpurun_out/${TAG}_C4_bench.json 2> gpurun_out/${TAG}_C4_bench.err
tail -1 gpurun_out/${TAG}_C4_bench.err; python -c "import json; d=json.loads(open('gpurun_out/${TAG}_C4_bench.json').read().strip().splitlines()[-1]); print('C4', d['value'], d['e2e']['value'], d['stages_ms'], d['roofline']['frac'], d['roofline']['kernel'], d['cpu_baseline']['value'])"
timeout 2400 python scripts/sweep_c5.py 100000000 100000 3 > gpurun_out/${TAG}_c5_sweep.jsonl 2> gpurun_out/${TAG}_c5_sweep.err
tail -2 gpurun_out/${TAG}_c5_sweep.err; cut -c1-250 gpurun_out/${TAG}_c5_sweep.jsonl
