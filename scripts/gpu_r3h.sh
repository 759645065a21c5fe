# narrow S8 sort key: GPU suite + A/B (TM_SCAN_VARIANT=14) at C2 / C3 / C4
TAG=${1:-r3h}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
S=$(date +%s); TM_FULL_SIZE=0 timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$? in $(( $(date +%s) - S )) s"; tail -1 gpurun_out/${TAG}_pytest.log
timeout 600 python scripts/ab.py C2 "14" "5000" 9 > gpurun_out/${TAG}_ab_C2.jsonl 2>&1; echo "ab C2 rc=$?"
timeout 900 python scripts/ab.py C3 "14" "5000" 5 > gpurun_out/${TAG}_ab_C3.jsonl 2>&1; echo "ab C3 rc=$?"
timeout 900 python scripts/ab.py C4 "14" "10000" 3 > gpurun_out/${TAG}_ab_C4.jsonl 2>&1; echo "ab C4 rc=$?"
