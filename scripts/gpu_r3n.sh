# pipelined CSR with the pinned-block size hint: e2e at C3 for 3 / 4 / 6 ranges, C4 at 4
TAG=${1:-r3n}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for P in 3 4 6; do
TM_PIPELINE=$P timeout 1200 python bench.py --steps 10 --warmup 3 --no-hbm --no-cpu-baseline > gpurun_out/${TAG}_C3_p$P.json 2> gpurun_out/${TAG}_C3_p$P.err; echo "bench p$P rc=$?"
done
timeout 1200 python bench.py --config C4 --steps 3 --warmup 2 --no-hbm --no-cpu-baseline > gpurun_out/${TAG}_C4_p4.json 2> gpurun_out/${TAG}_C4_p4.err; echo "bench C4 p4 rc=$?"
timeout 900 python bench.py --config C2 --steps 20 --warmup 5 --no-hbm --no-cpu-baseline > gpurun_out/${TAG}_C2.json 2> gpurun_out/${TAG}_C2.err; echo "bench C2 rc=$?"
