# one ncu --set full capture of k_scan per forced variant.  usage: bash scripts/gpu_ncu_var.sh <tag> "<variants>" [bench args]
TAG=${1:-nv}; VARS=${2:-"5 6"}; shift 2; ARGS="$*"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
for v in $VARS; do
  TM_SCAN_VARIANT=$v timeout 900 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:k_scan -s 3 -c 1 \
    -o gpurun_out/${TAG}_v${v} python bench.py --steps 1 --warmup 3 --no-cpu-baseline $ARGS > gpurun_out/${TAG}_v${v}.log 2>&1
  tail -1 gpurun_out/${TAG}_v${v}.log
done
