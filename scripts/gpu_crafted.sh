# sec. 4.4 crafted workload (C6/C7): exact mode, unique, and a MAX_P sweep at C6.
# usage: bash scripts/gpu_crafted.sh <tag>
TAG=${1:-crafted}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
run() {  # name, bench args
  local n=$1; shift
  timeout 600 python bench.py --steps 10 --warmup 3 --no-cpu-baseline "$@" > gpurun_out/${TAG}_$n.json 2> gpurun_out/${TAG}_$n.err
  python -c "import json; d=json.loads(open('gpurun_out/${TAG}_$n.json').read().strip().splitlines()[-1]); s=d['path_stats']; print('$n', round(d['value']/1e6,3), 'Mq/s e2e', round(d['e2e']['value']/1e6,3), 'scan', round(d['stages_ms']['scan_ms'],3), 'total', round(d['stages_ms']['total_ms'],3), 'parts', s['n_partitions'], 'cand', s['candidate_pairs'], 'checks', s['pair_checks'], 'pairs', s['result_pairs'], 'exact', s['exact_checked'], s['exact_kept'])" || tail -3 gpurun_out/${TAG}_$n.err
}
run C6_exact --config C6 --exact
run C7_exact --config C7 --exact
run C6_unique --config C6 --unique
for mp in 50000 20000 5000; do run C6_maxp$mp --config C6 --max-partition $mp; done
