cd $GRAFT_REPO_ROOT
export SHAPES="[(120,7200),(7200,120),(64,10000),(10000,64),(256,256),(64,64)]"
echo '[{}, {"IPT_TILE_GRP":1}]' > /tmp/v.json
for h in 0 1 2 3; do
  IPT_NVCC_EXTRA="-DIPT_ST_HINT=$h" python -m paper_conf_ppopp_sunggggh14_b200.build --force > /dev/null 2>&1
  echo "== hint $h" >> gpurun_out/sthint.txt
  VARIANTS_FILE=/tmp/v.json timeout 300 python tools/tile_big.py >> gpurun_out/sthint.txt 2>&1
  timeout 300 python bench.py --steps 6 --warmup 3 --no-e2e --no-cpu 2>/dev/null | python -c "import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('sweep', d['value'], {k:v['stage_gbs'] for k,v in d['per_shape'].items()})" >> gpurun_out/sthint.txt
done
