TAG=${1:-r2j}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
TM_FULL_SIZE=0 timeout 900 python -m pytest tests -m gpu -q -x -k "variant or fuzz or c1 or c2_full" > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/${TAG}_pytest.log
for UT in 4 8 16; do
  TM_UNIT_TARGET=$UT timeout 600 python scripts/ab.py C2 "14" "5000" 7 > gpurun_out/${TAG}_ab_C2_ut$UT.jsonl 2>&1
  TM_UNIT_TARGET=$UT timeout 900 python scripts/ab.py C3 "14" "5000" 5 > gpurun_out/${TAG}_ab_C3_ut$UT.jsonl 2>&1
  echo "ut=$UT done"
done
timeout 1500 python scripts/sweep_c5.py 100000000 100000 3 > gpurun_out/${TAG}_c5_sweep.jsonl 2> gpurun_out/${TAG}_c5.err; echo "c5 rc=$?"
for C in C6 C7; do timeout 900 python bench.py --config $C --steps 10 --warmup 3 --no-hbm > gpurun_out/${TAG}_${C}_bench.json 2> gpurun_out/${TAG}_${C}.err; echo "$C rc=$?"; done
