# session-3 first check: build, smoke, variant parity (incl. 16), A/B of 14 vs 16 at C2/C3/C4
TAG=${1:-r3a}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
TM_FULL_SIZE=0 timeout 900 python -m pytest tests -m gpu -q -x -k "variant or fuzz or c1 or c2_full" > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/${TAG}_pytest.log
timeout 600 python scripts/ab.py C2 "14,16" "5000" 7 > gpurun_out/${TAG}_ab_C2.jsonl 2>&1; echo "ab C2 rc=$?"
timeout 900 python scripts/ab.py C3 "14,16,14,16" "5000" 5 > gpurun_out/${TAG}_ab_C3.jsonl 2>&1; echo "ab C3 rc=$?"
timeout 900 python scripts/ab.py C4 "14,16" "10000" 3 > gpurun_out/${TAG}_ab_C4.jsonl 2>&1; echo "ab C4 rc=$?"
