# full-size configs on the GPU box: sampled parity + bench line
# usage: bash scripts/gpu_full.sh C3
CFG=${1:-C3}
mkdir -p gpurun_out
nproc; free -g | head -2
python -c "import __graft_entry__ as g; g.build()"
TM_FULL_SIZE=$CFG timeout 3000 python -m pytest tests/test_gpu_full.py -m gpu -x -q -s 2>&1 | tail -25
timeout 3000 python bench.py --config $CFG --steps 5 --warmup 3 --cpu-s 20 > gpurun_out/${CFG}_bench.json 2> gpurun_out/${CFG}_bench.err
tail -3 gpurun_out/${CFG}_bench.err; cat gpurun_out/${CFG}_bench.json
