# supplemental ncu capture of scan variant 8 at the bench configs (the tuner may pick 8 or 14);
# writes profiles/ncu_scan_traffic_<CFG>_v8.json for bench.py's traffic lookup
TAG=${1:-v8}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
BID=$(python -c "from paper_conf_eurosys_rogorapkmcc17_b200 import tagmatch as t; print(t.build_id())")
for CFG in C3 C4; do
  TM_SCAN_VARIANT=8 timeout 1500 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on \
    --nvtx --nvtx-include "bench_device/" -k regex:k_scan -s 3 -c 1 -o gpurun_out/${TAG}_${CFG}_scan \
    python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline --no-hbm > gpurun_out/${TAG}_${CFG}_ncu.log 2>&1
  echo "ncu $CFG rc=$?"
  python scripts/ncu_summary.py gpurun_out/${TAG}_${CFG}_scan.ncu-rep --config $CFG --build-id $BID --variant 8 \
    --json gpurun_out/${TAG}_ncu_scan_traffic_${CFG}_v8.json > gpurun_out/${TAG}_${CFG}_scan_ncu.txt 2>&1
done
