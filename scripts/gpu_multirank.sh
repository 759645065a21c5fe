# functional check of bench.py's N > 1 code paths on ONE GPU: 2 ranks share GPU 0,
# control plane over gloo (NCCL cannot place two ranks on one device).
python -c "import __graft_entry__ as g; g.build()"
TM_BENCH_PG=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29511 bench.py --gpus 2 --steps 3 --warmup 3 2> gpurun_out/mr.err | tail -2 | tee gpurun_out/mr.json
tail -3 gpurun_out/mr.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29512 bench.py --impl reference --gpus 2 --steps 2 --warmup 3 --ref-step-s 2 2> gpurun_out/mr_ref.err | tail -2
tail -3 gpurun_out/mr_ref.err
