# level-A block size A/B (TM_BLOCK_TILES 2 / 4 / 8) at C3 (5K, 200K), C4 (10K), C6
TAG=${1:-r3u}
mkdir -p gpurun_out
for BT in 8 4 2; do
  TM_NVCC_FLAGS="-DTM_BLOCK_TILES=$BT" python -m paper_conf_eurosys_rogorapkmcc17_b200._build --force > /dev/null 2>&1; echo "build $BT rc=$?"
  timeout 900 python scripts/ab.py C3 "14,8" "5000,200000" 3 > gpurun_out/${TAG}_C3_bt$BT.jsonl 2>&1; echo "C3 $BT rc=$?"
  timeout 900 python scripts/ab.py C4 "14" "10000" 3 > gpurun_out/${TAG}_C4_bt$BT.jsonl 2>&1; echo "C4 $BT rc=$?"
  AB_FILTER=1 timeout 600 python scripts/ab.py C6 "14" "0" 5 > gpurun_out/${TAG}_C6_bt$BT.jsonl 2>&1; echo "C6 $BT rc=$?"
done
python -m paper_conf_eurosys_rogorapkmcc17_b200._build --force > /dev/null 2>&1
