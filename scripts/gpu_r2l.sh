# r2l: bench.py's N > 1 path (2 ranks sharing one GPU, gloo control plane, replicated mode: the
# NCCL exchange cannot run with two ranks on one device), the reference arm under torchrun, and
# streaming latency vs batch timeout (Fig. 6 analogue) at C2 and C3.
TAG=${1:-r2l}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
TM_BENCH_PG=gloo timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29511 bench.py --gpus 2 --replicated --config C2 --steps 5 --warmup 3 > gpurun_out/${TAG}_mr.json 2> gpurun_out/${TAG}_mr.err
echo "multirank rc=$?"; tail -c 1500 gpurun_out/${TAG}_mr.json; tail -3 gpurun_out/${TAG}_mr.err
timeout 900 python -m torch.distributed.run --nnodes=1 --nproc-per-node 2 --master-addr 127.0.0.1 \
    --master-port 29512 bench.py --impl reference --gpus 2 --steps 2 --warmup 3 --ref-step-s 2 --config C2 > gpurun_out/${TAG}_mr_ref.json 2> gpurun_out/${TAG}_mr_ref.err
echo "multirank ref rc=$?"; tail -c 400 gpurun_out/${TAG}_mr_ref.json
timeout 1500 python scripts/stream_latency.py C2 2000000 400000 "100,250,500,1000,2000,5000" > gpurun_out/${TAG}_stream_C2.jsonl 2> gpurun_out/${TAG}_stream.err; echo "stream C2 rc=$?"
timeout 2400 python scripts/stream_latency.py C3 400000 300000 "1000,5000,20000,100000" > gpurun_out/${TAG}_stream_C3.jsonl 2>> gpurun_out/${TAG}_stream.err; echo "stream C3 rc=$?"
