# A/B: variant 14 (72 regs, 7 CTAs/SM) vs 17 (80 regs, 6 CTAs/SM)
TAG=${1:-r3i}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 600 python scripts/ab.py C2 "14,17" "5000" 7 > gpurun_out/${TAG}_ab_C2.jsonl 2>&1; echo "ab C2 rc=$?"
timeout 900 python scripts/ab.py C3 "14,17" "5000" 5 > gpurun_out/${TAG}_ab_C3.jsonl 2>&1; echo "ab C3 rc=$?"
