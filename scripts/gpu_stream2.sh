TAG=${1:-st}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python scripts/stream_latency.py C2 2000000 400000 "100,500,2000,5000,5000,10000" > gpurun_out/${TAG}_stream_C2.jsonl 2> gpurun_out/${TAG}_stream.err; echo "stream C2 rc=$?"
timeout 2400 python scripts/stream_latency.py C3 400000 300000 "1000,1000,5000,20000" > gpurun_out/${TAG}_stream_C3.jsonl 2>> gpurun_out/${TAG}_stream.err; echo "stream C3 rc=$?"
