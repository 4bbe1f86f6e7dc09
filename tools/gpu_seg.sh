cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
export PLANS='[(1800,7200,1800,180),(7200,1800,144,1800)]'
for m in "IPT_CYC_SEG=2" "IPT_CYC_SEG=2 IPT_SEG_DIAG=1" "IPT_CYC_SEG=2 IPT_SEG_DIAG=2" "IPT_CYC_SEG=2 IPT_SEG_DIAG=3"; do echo "$m" >> gpurun_out/plan_ab.txt; env $m timeout 600 python tools/plan_ab.py >> gpurun_out/plan_ab.txt 2>&1; done
IPT_CYC_SEG=2 timeout 300 /usr/local/cuda/bin/ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/seg_launches.csv python tools/plan_ab.py > /dev/null 2>&1
