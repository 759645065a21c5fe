# compile-time knob A/B on the final kernel at C3 / C2 (TM_NVCC_FLAGS rebuilds; the last build restores defaults)
TAG=${1:-r3t}
mkdir -p gpurun_out
for F in "" "-DTM_BLOCK_TILES=4" "-DTM_BLOCK_TILES=16" "-DTM_SUBW=64" "-DTM_CHUNK=512"; do
  N=$(echo "x$F" | tr -c 'a-zA-Z0-9' '_')
  TM_NVCC_FLAGS="$F" python -m paper_conf_eurosys_rogorapkmcc17_b200._build --force > /dev/null 2>&1; echo "build $F rc=$?"
  timeout 600 python scripts/ab.py C3 "14" "5000" 3 > gpurun_out/${TAG}_C3_${N}.jsonl 2>&1; echo "C3 $F rc=$?"
  timeout 300 python scripts/ab.py C2 "14" "5000" 7 > gpurun_out/${TAG}_C2_${N}.jsonl 2>&1; echo "C2 $F rc=$?"
done
python -m paper_conf_eurosys_rogorapkmcc17_b200._build --force > /dev/null 2>&1
