# pipelined CSR: e2e at C3 for 2 / 3 / 5 / 6 query ranges (r3l: 1 / 4 / 8)
TAG=${1:-r3m}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for P in 2 3 5 6; do
TM_PIPELINE=$P timeout 1200 python bench.py --steps 10 --warmup 3 --no-hbm --no-cpu-baseline > gpurun_out/${TAG}_C3_p$P.json 2> gpurun_out/${TAG}_C3_p$P.err; echo "bench p$P rc=$?"
done
TM_PIPELINE=1 timeout 1200 python bench.py --config C4 --steps 3 --warmup 2 --no-hbm --no-cpu-baseline > gpurun_out/${TAG}_C4_p1.json 2> gpurun_out/${TAG}_C4_p1.err; echo "bench C4 p1 rc=$?"
timeout 1200 python bench.py --config C4 --steps 3 --warmup 2 --no-hbm --no-cpu-baseline > gpurun_out/${TAG}_C4_p4.json 2> gpurun_out/${TAG}_C4_p4.err; echo "bench C4 p4 rc=$?"
