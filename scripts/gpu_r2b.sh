# r2b: parity of the new router + dense/IMAD variants, A/B of variants and MAX_P, HBM sweep by
# variant, compute-sanitizer logs.   usage: bash scripts/gpu_r2b.sh <tag>
TAG=${1:-r2b}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
TM_FULL_SIZE=0 timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/${TAG}_pytest.log
timeout 600 python scripts/ab.py C2 "5,8,0" "200000,50000,20000,5000" 7 > gpurun_out/${TAG}_ab_C2.jsonl 2>&1; echo "ab C2 rc=$?"
timeout 900 python scripts/ab.py C3 "5,8" "200000,50000,20000,10000,5000" 5 > gpurun_out/${TAG}_ab_C3.jsonl 2>&1; echo "ab C3 rc=$?"
HBM_VARIANTS=auto,5,9,10,11,12 timeout 900 python scripts/hbm_sweep.py 100000000 2 > gpurun_out/${TAG}_hbm.jsonl 2> gpurun_out/${TAG}_hbm.err; echo "hbm rc=$?"
for T in memcheck racecheck synccheck; do
  N=100000; [ $T != memcheck ] && N=20000
  timeout 1200 /usr/local/cuda/bin/compute-sanitizer --tool $T --error-exitcode 99 python scripts/sanitize.py \
    0,1,2,3,4,5,6,7,8,9,10,11,12 $N > gpurun_out/${TAG}_sanitize_${T}.log 2>&1; echo "sanitize $T rc=$?"; tail -3 gpurun_out/${TAG}_sanitize_${T}.log
done
