# 128-row level-A blocks as variants 17 / 18: parity subset, then A/B vs 14 / 8
TAG=${1:-r3v}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
TM_FULL_SIZE=0 timeout 1500 python -m pytest tests -m gpu -q -x -k "variant or fuzz or c1 or c2 or tuning" > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/${TAG}_pytest.log
timeout 900 python scripts/ab.py C3 "14,17,8,18" "5000" 3 > gpurun_out/${TAG}_ab_C3.jsonl 2>&1; echo "C3 rc=$?"
timeout 900 python scripts/ab.py C4 "14,17,8,18" "10000" 3 > gpurun_out/${TAG}_ab_C4.jsonl 2>&1; echo "C4 rc=$?"
timeout 600 python scripts/ab.py C2 "14,17,8,18,auto" "5000" 7 > gpurun_out/${TAG}_ab_C2.jsonl 2>&1; echo "C2 rc=$?"
