# bucket merge (S8 by query buckets) vs the LSD radix merge: GPU suite + C3/C4 A/B
TAG=${1:-r3d}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -2
S=$(date +%s); TM_FULL_SIZE=0 timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$? in $(( $(date +%s) - S )) s"; tail -2 gpurun_out/${TAG}_pytest.log
timeout 900 python scripts/ab.py C3 "14" "5000" 5 > gpurun_out/${TAG}_ab_C3_bucket.jsonl 2>&1; echo "ab C3 rc=$?"
TM_RADIX_MERGE=1 timeout 900 python scripts/ab.py C3 "14" "5000" 5 > gpurun_out/${TAG}_ab_C3_radix.jsonl 2>&1; echo "ab C3 radix rc=$?"
timeout 900 python scripts/ab.py C4 "14" "10000" 3 > gpurun_out/${TAG}_ab_C4_bucket.jsonl 2>&1; echo "ab C4 rc=$?"
timeout 600 python scripts/ab.py C2 "14" "5000" 7 > gpurun_out/${TAG}_ab_C2_bucket.jsonl 2>&1; echo "ab C2 rc=$?"
