# A/B of prebuilt library variants (exp_libs/libtagmatch_<name>.so): C2 bench per library, with the
# sources' mtimes older than the copied library so nothing is rebuilt.  usage: bash scripts/gpu_lib_ab.sh <tag> "<names>" [bench args]
TAG=${1:-lab}; NAMES=${2:-""}; shift 2; EXTRA="$*"
mkdir -p gpurun_out
LIB=paper_conf_eurosys_rogorapkmcc17_b200/libtagmatch.so
cp $LIB /tmp/libtagmatch_orig.so
for n in $NAMES; do
  cp exp_libs/libtagmatch_$n.so $LIB; touch $LIB
  timeout 900 python bench.py --steps 10 --warmup 3 --no-cpu-baseline $EXTRA > gpurun_out/${TAG}_$n.json 2> gpurun_out/${TAG}_$n.err
  python -c "import json; d=json.loads(open('gpurun_out/${TAG}_$n.json').read().strip().splitlines()[-1]); print('$n', d['config']['workload'], round(d['value']/1e6,3), 'Mq/s scan', round(d['stages_ms']['scan_ms'],3), 'frac', round(d['roofline']['frac'],3), d['path_stats']['tile_tests'], d['path_stats']['pair_checks'])" || tail -3 gpurun_out/${TAG}_$n.err
done
cp /tmp/libtagmatch_orig.so $LIB; touch $LIB
