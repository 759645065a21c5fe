TAG=${1:-r2o}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
TM_ROUTE=1 TM_FULL_SIZE=0 timeout 1200 python -m pytest tests -m gpu -q -x -k "group or store or shard or fuzz or c1 or c2" > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest(route t) rc=$?"; tail -2 gpurun_out/${TAG}_pytest.log
for R in 0 1; do
  TM_ROUTE=$R timeout 600 python scripts/ab.py C2 "14" "5000" 7 > gpurun_out/${TAG}_ab_C2_r$R.jsonl 2>&1
  TM_ROUTE=$R timeout 900 python scripts/ab.py C3 "14" "5000" 5 > gpurun_out/${TAG}_ab_C3_r$R.jsonl 2>&1
  TM_ROUTE=$R timeout 900 python scripts/ab.py C4 "14" "10000" 3 > gpurun_out/${TAG}_ab_C4_r$R.jsonl 2>&1
  echo "route $R done"
done
TM_ROUTE=1 HBM_B=1,4,16 timeout 900 python scripts/hbm_sweep.py 100000000 2 > gpurun_out/${TAG}_hbm.jsonl 2> gpurun_out/${TAG}_hbm.err; echo "hbm rc=$?"
