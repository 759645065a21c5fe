# one ncu --set full capture of k_scan at C3 and C4 in the bench configuration (after the tuning
# calls, the warm-up and one timed step), for the roofline's traffic at those sizes.
# usage: bash scripts/gpu_ncu_big.sh <tag>
TAG=${1:-nb}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
for C in C3 C4; do
  timeout 1800 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:k_scan -s 10 -c 1 \
    -o gpurun_out/${TAG}_${C}_scan python bench.py --config $C --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_${C}_ncu.log 2>&1
  tail -1 gpurun_out/${TAG}_${C}_ncu.log
done
