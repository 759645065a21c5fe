TAG=${1:-r2h}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
TM_FULL_SIZE=0 timeout 1200 python -m pytest tests -m gpu -q -x -k "variant or fuzz or c1 or group or store or shard" > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/${TAG}_pytest.log
timeout 900 python scripts/ab.py C3 "14" "5000,10000" 5 > gpurun_out/${TAG}_ab_C3.jsonl 2>&1; echo "ab C3 rc=$?"
timeout 900 python scripts/ab.py C4 "14" "10000" 3 > gpurun_out/${TAG}_ab_C4.jsonl 2>&1; echo "ab C4 rc=$?"
HBM_B=8,16,32,64 HBM_VARIANTS=13,15,9 timeout 900 python scripts/hbm_sweep.py 100000000 2 > gpurun_out/${TAG}_hbm.jsonl 2> gpurun_out/${TAG}_hbm.err; echo "hbm rc=$?"
