TAG=${1:-r2f}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
TM_FULL_SIZE=0 timeout 1200 python -m pytest tests -m gpu -q -x -k "store or group or variant or fuzz or c1" > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -2 gpurun_out/${TAG}_pytest.log
for BV in "16 13" "32 13" "64 9"; do set -- $BV
  timeout 600 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:k_dense -s 2 -c 1 \
    -o gpurun_out/${TAG}_dense_B$1_v$2 python scripts/dense_probe.py $1 $2 > gpurun_out/${TAG}_dense_B$1.log 2>&1; echo "ncu dense B=$1 rc=$?"
done
timeout 900 python scripts/build_time.py 1000000,5000000 > gpurun_out/${TAG}_build_time.jsonl 2>&1; echo "build_time rc=$?"
for T in memcheck racecheck synccheck; do
  N=100000; [ $T != memcheck ] && N=20000
  timeout 1500 /usr/local/cuda/bin/compute-sanitizer --tool $T --error-exitcode 99 python scripts/sanitize.py \
    0,5,6,7,8,9,10,11,12,13,14,15 $N > gpurun_out/${TAG}_sanitize_${T}.log 2>&1; echo "sanitize $T rc=$?"; tail -2 gpurun_out/${TAG}_sanitize_${T}.log
done
