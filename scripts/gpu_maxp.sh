# MAX_P sweep (Fig. 7 analogue) on a config
CFG=${1:-C2}
python -c "import __graft_entry__ as g; g.build()"
for mp in 200000 50000 20000 5000 1000; do
  timeout 1200 python bench.py --config $CFG --steps 5 --warmup 3 --no-cpu-baseline --max-partition $mp > gpurun_out/maxp_${CFG}_$mp.json 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/maxp_${CFG}_$mp.json').read().strip().splitlines()[-1]); s=d['path_stats']; print($mp, round(d['value']), 'scan_ms', round(d['roofline']['kernel_ms'],3), 'route_ms', round(d['stages_ms']['route_ms'],3), 'P', s['n_partitions'], 'cand', s['candidate_pairs'], 'checks', s['pair_checks'])"
done
