# C4 full-size parity + bench line, then the C5 sweep (one GPU)
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
TM_FULL_SIZE=C4 timeout 3000 python -m pytest tests/test_gpu_full.py -m gpu -x -q -s 2>&1 | tail -12
timeout 3000 python bench.py --config C4 --steps 3 --warmup 3 --cpu-s 20 > gpurun_out/C4_bench.json 2> gpurun_out/C4_bench.err
tail -2 gpurun_out/C4_bench.err; cat gpurun_out/C4_bench.json
timeout 3000 python scripts/sweep_c5.py 100000000 100000 3 > gpurun_out/c5_sweep.jsonl 2> gpurun_out/c5_sweep.err
tail -2 gpurun_out/c5_sweep.err; cat gpurun_out/c5_sweep.jsonl | cut -c1-300
