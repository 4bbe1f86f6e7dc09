cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ncu
for sh in "64 16384" "240 7200" "7200 400" "9998 128"; do
  tag=$(echo $sh | tr ' ' x)
  timeout 600 ncu --set full --import-source on --clock-control none -k regex:tile_group --launch-skip 1 -c 1 -o gpurun_out/ncu/tile_$tag -f python tools/tile_one.py $sh 3 > /dev/null 2>&1
done
ls -la gpurun_out/ncu
