# ncu --set full of k_scan (variant 14) at the bench configs C3 / C4: the committed per-config traffic
# json carries this build's id.   usage: bash scripts/gpu_ncu_final.sh <tag> [racecheck]
TAG=${1:-ncu}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
BID=$(python -c "from paper_conf_eurosys_rogorapkmcc17_b200 import tagmatch as t; print(t.build_id())")
for CFG in C3 C4; do
  TM_SCAN_VARIANT=14 timeout 1500 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on \
    -k regex:k_scan -s 6 -c 1 -o gpurun_out/${TAG}_${CFG}_scan \
    python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline --no-hbm > gpurun_out/${TAG}_${CFG}_ncu.log 2>&1
  echo "ncu $CFG rc=$?"
  python scripts/ncu_summary.py gpurun_out/${TAG}_${CFG}_scan.ncu-rep --config $CFG --build-id $BID --variant 14 \
    --json gpurun_out/${TAG}_ncu_scan_traffic_${CFG}.json > gpurun_out/${TAG}_${CFG}_scan_ncu.txt 2>&1
  head -3 gpurun_out/${TAG}_${CFG}_scan_ncu.txt
done
if [ "${2:-}" = "racecheck" ]; then
  timeout 2700 compute-sanitizer --tool racecheck --error-exitcode 99 python scripts/sanitize.py 0,5,6,7,8,9,10,11,12,13,14,15 10000 > gpurun_out/${TAG}_sanitize_racecheck.log 2>&1; echo "racecheck rc=$?"; tail -1 gpurun_out/${TAG}_sanitize_racecheck.log
fi
