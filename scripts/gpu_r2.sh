# round-2 check-in run: build + smoke, INT-peak microbenchmark, GPU tests, one ncu --set full
# capture of k_scan at the bench config (summary with build id + variant, so the bench line's
# roofline.traffic is from the same kernels), then the default bench line.
# usage: bash scripts/gpu_r2.sh <tag> [tests: all|none|<pytest -k expr>] [config]
TAG=${1:-r2}
T=${2:-all}
CFG=${3:-C3}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
./build/int_peak > gpurun_out/${TAG}_int_peak.json 2>&1; cat gpurun_out/${TAG}_int_peak.json
if [ "$T" != "none" ]; then
  S=$(date +%s)
  if [ "$T" = "all" ]; then timeout 1500 python -m pytest tests -m gpu -x -q -s > gpurun_out/${TAG}_pytest.log 2>&1;
  else timeout 1500 python -m pytest tests -m gpu -x -q -s -k "$T" > gpurun_out/${TAG}_pytest.log 2>&1; fi
  echo "pytest rc=$? in $(( $(date +%s) - S )) s"; tail -3 gpurun_out/${TAG}_pytest.log
fi
BID=$(python -c "from paper_conf_eurosys_rogorapkmcc17_b200 import tagmatch as t; print(t.build_id())")
VAR=${TM_NCU_VARIANT:-5}
TM_SCAN_VARIANT=$VAR timeout 1200 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on \
  -k regex:k_scan -s 10 -c 1 -o gpurun_out/${TAG}_${CFG}_scan \
  python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline --no-hbm > gpurun_out/${TAG}_ncu.log 2>&1
echo "ncu rc=$?"
python scripts/ncu_summary.py gpurun_out/${TAG}_${CFG}_scan.ncu-rep --config $CFG --build-id $BID --variant $VAR \
  --json profiles/ncu_scan_traffic_${CFG}.json > gpurun_out/${TAG}_${CFG}_scan_ncu.txt 2>&1
cp profiles/ncu_scan_traffic_${CFG}.json gpurun_out/${TAG}_ncu_scan_traffic_${CFG}.json
head -30 gpurun_out/${TAG}_${CFG}_scan_ncu.txt
timeout 1200 python bench.py --config $CFG --steps 10 --warmup 3 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err
echo "bench rc=$?"; tail -3 gpurun_out/${TAG}_bench.err; cat gpurun_out/${TAG}_bench.json
