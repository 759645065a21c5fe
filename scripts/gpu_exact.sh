python -c "import __graft_entry__ as g; g.build()"
for cfg in C2 C3; do
for ex in "" "--exact"; do
  timeout 1500 python bench.py --config $cfg --steps 5 --warmup 3 --no-cpu-baseline $ex > gpurun_out/exact.json 2> gpurun_out/exact.err
  python -c "import json; d=json.loads(open('gpurun_out/exact.json').read().strip().splitlines()[-1]); s=d['path_stats']; print('$cfg', '$ex', round(d['value']), 'ms', round(d['ms_per_step'],2), 'scan', round(d['roofline']['kernel_ms'],2), 'matched', s['matched_sets'], 'emitted', s['emitted_pairs'], 'result', s['result_pairs'], 'checked', s['exact_checked'], 'kept', s['exact_kept'])" || tail -5 gpurun_out/exact.err
done; done
