# ncu full capture of one k_scan launch at a given config (after warm-up launches)
# usage: bash scripts/gpu_profile_cfg.sh <tag> <config>
TAG=$1; CFG=$2
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()"
timeout 2400 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:k_scan -s 3 -c 1 \
    -o gpurun_out/${TAG}_scan python bench.py --config $CFG --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/${TAG}_full.log 2>&1
tail -3 gpurun_out/${TAG}_full.log
