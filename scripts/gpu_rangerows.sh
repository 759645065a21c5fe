# work-item size sweep (TM_RANGE_ROWS) at C2 and C3: bench q/s and scan ms
python -c "import __graft_entry__ as g; g.build()"
timeout 600 python -m pytest tests -m gpu -x -q -k "c1_single or small or c2_full" 2>&1 | tail -1
for cfg in C2 C3; do
for rr in 4096 8192 16384 32768; do
  TM_RANGE_ROWS=$rr timeout 900 python bench.py --config $cfg --steps 5 --warmup 3 --no-cpu-baseline > gpurun_out/rr_${cfg}_$rr.json 2>&1
  python -c "import json; d=json.loads(open('gpurun_out/rr_${cfg}_$rr.json').read().strip().splitlines()[-1]); print('$cfg', $rr, round(d['value']), 'scan_ms', round(d['roofline']['kernel_ms'],3), d['path_stats']['work_items'])"
done
done
