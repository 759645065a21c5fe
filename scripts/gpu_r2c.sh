# r2c: parity (variants incl. 13/14, fuzz, C1/C2), A/B C2/C3 of 5/8/14 at 200K and auto MAX_P,
# dense HBM sweep points, memcheck of the new kernels.   usage: bash scripts/gpu_r2c.sh <tag>
TAG=${1:-r2c}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
TM_FULL_SIZE=0 timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -3 gpurun_out/${TAG}_pytest.log
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 99 python scripts/sanitize.py 9,10,13,14 20000 > gpurun_out/${TAG}_memcheck.log 2>&1; echo "memcheck rc=$?"; tail -2 gpurun_out/${TAG}_memcheck.log
timeout 600 python scripts/ab.py C2 "5,8,14" "200000,5000" 7 > gpurun_out/${TAG}_ab_C2.jsonl 2>&1; echo "ab C2 rc=$?"
timeout 900 python scripts/ab.py C3 "5,8,14" "200000,10000" 5 > gpurun_out/${TAG}_ab_C3.jsonl 2>&1; echo "ab C3 rc=$?"
HBM_B=8,16,32,64,256 HBM_VARIANTS=9,13,10 timeout 900 python scripts/hbm_sweep.py 100000000 2 > gpurun_out/${TAG}_hbm.jsonl 2> gpurun_out/${TAG}_hbm.err; echo "hbm rc=$?"
