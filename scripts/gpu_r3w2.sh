# bench lines of the final build with its committed ncu captures in place (traffic in the line)
TAG=${1:-r3w2}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1200 python bench.py --steps 20 --warmup 5 > gpurun_out/${TAG}_bench.json 2> gpurun_out/${TAG}_bench.err; echo "bench C3 rc=$?"
timeout 1500 python bench.py --config C4 --steps 5 --warmup 3 --no-hbm > gpurun_out/${TAG}_C4_bench.json 2> gpurun_out/${TAG}_C4_bench.err; echo "bench C4 rc=$?"
