TAG=${1:-r3e}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -2
for CFG in "C3 5000"; do
timeout 900 /usr/local/cuda/bin/ncu --profile-from-start off --metrics gpu__time_duration.sum --clock-control none --csv \
  --log-file gpurun_out/${TAG}_stages.csv python scripts/stage_probe.py $CFG > gpurun_out/${TAG}_stages.log 2>&1; echo "ncu rc=$?"
done
