# final-build evidence: C5 query-size sweep at 100M sets and C7 bench line
TAG=${1:-r3s}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
timeout 1500 python scripts/sweep_c5.py 100000000 100000 3 > gpurun_out/${TAG}_c5_sweep.jsonl 2> gpurun_out/${TAG}_c5.err; echo "c5 rc=$?"
timeout 900 python bench.py --config C7 --steps 10 --warmup 3 --no-hbm > gpurun_out/${TAG}_C7_bench.json 2> gpurun_out/${TAG}_C7_bench.err; echo "bench C7 rc=$?"
