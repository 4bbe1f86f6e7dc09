# A/B of two tile_onchip.cu variants (tools/ab/tile_onchip_{A,B}.cu) on tools/tile_big.py
cd $GRAFT_REPO_ROOT
cp paper_conf_ppopp_sunggggh14_b200/csrc/tile_onchip.cu /tmp/cur.cu
for v in A B A B; do
  cp tools/ab/tile_onchip_$v.cu paper_conf_ppopp_sunggggh14_b200/csrc/tile_onchip.cu
  python -m paper_conf_ppopp_sunggggh14_b200.build --force > /tmp/build_$v.log 2>&1 || { echo "build $v failed"; tail -5 /tmp/build_$v.log; }
  echo "== $v" >> gpurun_out/ab.txt
  VARIANTS_FILE=${VARIANTS_FILE:-tools/variants_tile.json} timeout 600 python tools/tile_big.py >> gpurun_out/ab.txt 2>&1
done
cp /tmp/cur.cu paper_conf_ppopp_sunggggh14_b200/csrc/tile_onchip.cu
