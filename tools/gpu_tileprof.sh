cd $GRAFT_REPO_ROOT
M="gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_sectors_srcunit_tex_op_write.sum,dram__throughput.avg.pct_of_peak_sustained_elapsed,lts__t_sectors_srcunit_tex_op_read_lookup_hit.sum,lts__t_sectors_srcunit_tex_op_write_lookup_hit.sum"
for cfg in "" "IPT_TILE_GRP=1 IPT_TILE_GRP_K=16" "IPT_TILE_GRP=1 IPT_TILE_GRP_K=16 IPT_TILE_GRP_G=7 IPT_TILE_GRP_NOBAR=1" "IPT_TILE_GRP=1 IPT_TILE_GRP_K=16 IPT_TILE_GRP_NOBAR=1"; do
  for sh in "120 7200" "64 10000"; do
    echo "== $cfg / $sh" >> gpurun_out/tileprof.txt
    env $cfg timeout 300 ncu --metrics $M --clock-control none -k regex:tile --csv python tools/tile_one.py $sh 2 2>/dev/null | grep -v "^==PROF" | python -c "
import sys,csv
rows=list(csv.reader(sys.stdin))
hdr=None
for r in rows:
    if r and r[0]=='ID': hdr=r; continue
    if hdr and len(r)==len(hdr) and r[hdr.index('ID')]=='1':
        print(r[hdr.index('Metric Name')], r[hdr.index('Metric Value')])
" >> gpurun_out/tileprof.txt
  done
done
