# A/B of 14 vs 16 (branch-free level B / full check), parity subset first
TAG=${1:-r3c}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
TM_FULL_SIZE=0 timeout 900 python -m pytest tests -m gpu -q -x -k "every_scan_variant" > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/${TAG}_pytest.log
timeout 600 python scripts/ab.py C2 "14,16" "5000" 7 > gpurun_out/${TAG}_ab_C2.jsonl 2>&1; echo "ab C2 rc=$?"
timeout 900 python scripts/ab.py C3 "14,16,14,16" "5000" 5 > gpurun_out/${TAG}_ab_C3.jsonl 2>&1; echo "ab C3 rc=$?"
