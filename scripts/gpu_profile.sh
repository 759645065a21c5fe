# ncu evidence for the scan kernel: launch list (per-launch device times) and one --set full capture.
# usage: bash scripts/gpu_profile.sh <tag> [bench args...]
set -x
TAG=${1:-r1}; shift
ARGS="$@"
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
NCU=/usr/local/cuda/bin/ncu
timeout 900 $NCU --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/${TAG}_launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline $ARGS > gpurun_out/${TAG}_launches_bench.log 2>&1
timeout 1200 $NCU --set full --clock-control none --import-source on -k regex:k_scan -s 3 -c 1 \
    -o gpurun_out/${TAG}_scan python bench.py --steps 1 --warmup 3 --no-cpu-baseline $ARGS > gpurun_out/${TAG}_full.log 2>&1
tail -5 gpurun_out/${TAG}_full.log
ls -la gpurun_out
