# compare layouts (paper lexicographic+prefix vs balanced splits + AND masks) at a config
CFG=${1:-C2}
python -c "import __graft_entry__ as g; g.build()"
if [ "$CFG" = "C2" ]; then timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -3 > gpurun_out/layout_tests.txt; cat gpurun_out/layout_tests.txt; fi
for args in "--tile-filter 0 --row-order 0" "--tile-filter 1 --row-order 0" "--tile-filter 1 --row-order 1"; do
  timeout 2400 python bench.py --config $CFG --steps 5 --warmup 3 --no-cpu-baseline $args > gpurun_out/layout.json 2> gpurun_out/layout.err
  python -c "import json; d=json.loads(open('gpurun_out/layout.json').read().strip().splitlines()[-1]); s=d['path_stats']; print('$args', round(d['value']), 'scan_ms', round(d['roofline']['kernel_ms'],2), 'tests', s['tile_tests'], 'checks', s['pair_checks'], 'build_s', round(d['build_s'],1))"
done
