# knob sweep on the final kernel at C3 (MAX_P 5K, variant 14): TM_RANGE_ROWS x TM_UNIT_TARGET
TAG=${1:-r3r}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" 2>&1 | tail -1
for RR in 16384 32768 65536; do for UT in 4 8 16; do
  TM_RANGE_ROWS=$RR TM_UNIT_TARGET=$UT timeout 600 python scripts/ab.py C3 "14" "5000" 3 > gpurun_out/${TAG}_rr${RR}_ut${UT}.jsonl 2>&1; echo "rr $RR ut $UT rc=$?"
done; done
