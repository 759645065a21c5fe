# final check-in of a round: full GPU suite (SKIP_PYTEST=1 skips), ncu of the bench configs (traffic of this
# build), NVTX-filtered launch list, default bench line (C3) + C2 / C4 / C6 lines, the HBM sweep,
# the reference arm, per-kernel stage times.  compute-sanitizer is closed on the pool (session 3).  usage: bash scripts/gpu_final.sh <tag>
TAG=${1:-final}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
S=$(date +%s); [ -n "$SKIP_PYTEST" ] || timeout 1500 python -m pytest tests -m gpu -q -s > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$? in $(( $(date +%s) - S )) s"; tail -2 gpurun_out/${TAG}_pytest.log
BID=$(python -c "from paper_conf_eurosys_rogorapkmcc17_b200 import tagmatch as t; print(t.build_id())")
for CFG in C3 C4; do for V in ${NCU_VARIANTS:-17 18}; do
  TM_SCAN_VARIANT=$V timeout 1500 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on \
    --nvtx --nvtx-include "bench_device/" -k regex:k_scan -s 3 -c 1 -o gpurun_out/${TAG}_${CFG}_v${V}_scan \
    python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline --no-hbm > gpurun_out/${TAG}_${CFG}_v${V}_ncu.log 2>&1
  echo "ncu $CFG v$V rc=$?"
  python scripts/ncu_summary.py gpurun_out/${TAG}_${CFG}_v${V}_scan.ncu-rep --config $CFG --build-id $BID --variant $V \
    --json gpurun_out/${TAG}_ncu_scan_traffic_${CFG}_v${V}.json > gpurun_out/${TAG}_${CFG}_v${V}_scan_ncu.txt 2>&1
  cp gpurun_out/${TAG}_ncu_scan_traffic_${CFG}_v${V}.json profiles/ncu_scan_traffic_${CFG}_v${V}.json 2>/dev/null  # the bench lines below read it
done; done
timeout 900 /usr/local/cuda/bin/ncu --nvtx --nvtx-include "bench_device/" --metrics gpu__time_duration.sum --clock-control none \
  -c 200 --csv --log-file gpurun_out/${TAG}_launches.csv python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-hbm > /dev/null 2>&1; echo "launches rc=$?"
timeout 1200 python bench.py --steps 20 --warmup 5 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench C3 rc=$?"; tail -1 gpurun_out/${TAG}_bench.err
timeout 900 python bench.py --config C2 --steps 20 --warmup 5 --no-hbm > gpurun_out/${TAG}_C2_bench.json 2> gpurun_out/${TAG}_C2_bench.err; echo "bench C2 rc=$?"
timeout 1500 python bench.py --config C4 --steps 5 --warmup 3 --no-hbm > gpurun_out/${TAG}_C4_bench.json 2> gpurun_out/${TAG}_C4_bench.err; echo "bench C4 rc=$?"
timeout 900 python bench.py --config C6 --steps 10 --warmup 3 --no-hbm > gpurun_out/${TAG}_C6_bench.json 2> gpurun_out/${TAG}_C6_bench.err; echo "bench C6 rc=$?"
timeout 900 python scripts/hbm_sweep.py 100000000 2 > gpurun_out/${TAG}_hbm.jsonl 2> gpurun_out/${TAG}_hbm.err; echo "hbm rc=$?"
timeout 900 python bench.py --impl reference --steps 20 --warmup 5 > gpurun_out/${TAG}_reference.json 2> gpurun_out/${TAG}_reference.err; echo "reference rc=$?"
timeout 900 /usr/local/cuda/bin/ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${TAG}_stages_C3.csv python scripts/stage_probe.py C3 5000 > gpurun_out/${TAG}_stages_C3.log 2>&1; echo "stages rc=$?"
