# full default GPU suite (incl. full-size C3 / C4 at auto MAX_P and 200K, C5, C6 / C7)
TAG=${1:-r3j}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -1
S=$(date +%s); timeout 2400 python -m pytest tests -m gpu -q -s > gpurun_out/${TAG}_pytest.log 2>&1; echo "pytest rc=$? in $(( $(date +%s) - S )) s"; tail -3 gpurun_out/${TAG}_pytest.log
