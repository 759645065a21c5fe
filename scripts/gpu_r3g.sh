TAG=${1:-r3g}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
S=$(date +%s); TM_FULL_SIZE=0 timeout 1500 python -m pytest tests -m gpu -q -x > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$? in $(( $(date +%s) - S )) s"; tail -3 gpurun_out/${TAG}_pytest.log
