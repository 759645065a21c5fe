# ncu capture of k_scan for a scan variant: bash scripts/gpu_profile_var.sh <tag> <variant>
python -c "import __graft_entry__ as g; g.build()"
TM_SCAN_VARIANT=$2 timeout 900 python -m pytest tests -m gpu -x -q -k "c1_single or edge or c2_full or overflow or small" 2>&1 | tail -2
TM_SCAN_VARIANT=$2 timeout 1200 /usr/local/cuda/bin/ncu --set full --clock-control none --import-source on -k regex:k_scan -s 3 -c 1 \
    -o gpurun_out/$1_scan python bench.py --steps 1 --warmup 3 --no-cpu-baseline > gpurun_out/$1_full.log 2>&1
tail -2 gpurun_out/$1_full.log
