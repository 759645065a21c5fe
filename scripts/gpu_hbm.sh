python -c "import __graft_entry__ as g; g.build()"
timeout 1200 python -m pytest tests -m gpu -x -q -k "small_batches or edge or c1_single or empty" 2>&1 | tail -2
timeout 3000 python scripts/hbm_sweep.py ${1:-100000000} ${2:-2} > gpurun_out/hbm_sweep.jsonl 2> gpurun_out/hbm_sweep.err
tail -3 gpurun_out/hbm_sweep.err; cut -c1-200 gpurun_out/hbm_sweep.jsonl
