# pre-check pass statistics (diagnostic variant 17) at C2 / C3
TAG=${1:-r3b}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
timeout 600 python scripts/ab.py C2 "17" "5000" 1 > gpurun_out/${TAG}_dbg_C2.txt 2>&1; echo "C2 rc=$?"
timeout 900 python scripts/ab.py C3 "17" "5000" 1 > gpurun_out/${TAG}_dbg_C3.txt 2>&1; echo "C3 rc=$?"
