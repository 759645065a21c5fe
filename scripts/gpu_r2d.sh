# r2d: parity incl. in-process multi-GPU groups; A/B 5/8/14 (lazy rows); C4 MAX_P; dense sweep; bench
TAG=${1:-r2d}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
TM_FULL_SIZE=0 timeout 1200 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/${TAG}_pytest.log
timeout 600 python scripts/ab.py C2 "5,8,14" "200000,5000" 7 > gpurun_out/${TAG}_ab_C2.jsonl 2>&1; echo "ab C2 rc=$?"
timeout 900 python scripts/ab.py C3 "5,8,14" "200000,10000" 5 > gpurun_out/${TAG}_ab_C3.jsonl 2>&1; echo "ab C3 rc=$?"
timeout 1200 python scripts/ab.py C4 "8,14" "200000,30000,10000" 3 > gpurun_out/${TAG}_ab_C4.jsonl 2>&1; echo "ab C4 rc=$?"
HBM_B=8,16,32,64 HBM_VARIANTS=9,13 timeout 900 python scripts/hbm_sweep.py 100000000 2 > gpurun_out/${TAG}_hbm.jsonl 2> gpurun_out/${TAG}_hbm.err; echo "hbm rc=$?"
timeout 1200 python bench.py --steps 10 --warmup 3 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench rc=$?"; tail -2 gpurun_out/${TAG}_bench.err
