python -c "import __graft_entry__ as g; g.build()"
timeout 1500 python scripts/stream_latency.py C2 2000000 400000 "100,250,500,1000,2000,5000" > gpurun_out/stream_C2.jsonl 2> gpurun_out/stream.err
timeout 2400 python scripts/stream_latency.py C3 300000 300000 "1000,5000,20000,100000,300000" > gpurun_out/stream_C3.jsonl 2>> gpurun_out/stream.err
tail -3 gpurun_out/stream.err; cut -c1-330 gpurun_out/stream_C2.jsonl gpurun_out/stream_C3.jsonl
