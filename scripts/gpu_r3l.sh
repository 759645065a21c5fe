# pipelined CSR: parity tests, then the e2e bench at C3 with and without the pipeline
TAG=${1:-r3l}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
TM_FULL_SIZE=0 timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$?"; tail -1 gpurun_out/${TAG}_pytest.log
TM_PIPELINE=1 timeout 1200 python bench.py --steps 10 --warmup 3 --no-hbm --no-cpu-baseline > gpurun_out/${TAG}_C3_p1.json 2> gpurun_out/${TAG}_C3_p1.err; echo "bench p1 rc=$?"
timeout 1200 python bench.py --steps 10 --warmup 3 --no-hbm --no-cpu-baseline > gpurun_out/${TAG}_C3_p4.json 2> gpurun_out/${TAG}_C3_p4.err; echo "bench p4 rc=$?"
TM_PIPELINE=8 timeout 1200 python bench.py --steps 10 --warmup 3 --no-hbm --no-cpu-baseline > gpurun_out/${TAG}_C3_p8.json 2> gpurun_out/${TAG}_C3_p8.err; echo "bench p8 rc=$?"
