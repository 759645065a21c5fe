python -c "import __graft_entry__ as g; g.build(); g.smoke()" 2>&1 | tail -3
timeout 1800 python -m pytest tests -m gpu -x -q ${1:+-k "$1"} 2>&1 | tail -25
