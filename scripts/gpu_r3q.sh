# item filter (variant 17) vs 14 / 8: parity, then A/B at C2 / C3 (5K and 200K) / C4
TAG=${1:-r3q}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
TM_FULL_SIZE=0 timeout 1500 python -m pytest tests -m gpu -q -x -k "variant or fuzz or c1 or c2" > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/${TAG}_pytest.log
timeout 600 python scripts/ab.py C2 "14,17" "5000,200000" 7 > gpurun_out/${TAG}_ab_C2.jsonl 2>&1; echo "ab C2 rc=$?"
timeout 1200 python scripts/ab.py C3 "14,17,8" "5000,200000" 5 > gpurun_out/${TAG}_ab_C3.jsonl 2>&1; echo "ab C3 rc=$?"
timeout 1200 python scripts/ab.py C4 "14,17" "10000" 3 > gpurun_out/${TAG}_ab_C4.jsonl 2>&1; echo "ab C4 rc=$?"
