cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
export PLANS='[(12800,15000,256,15000),(7200,18000,7200,500),(18000,7200,240,7200),(9998,12288,9998,192),(12288,9998,192,9998),(14803,8192,14803,256),(7200,18000,7200,240)]'
for m in "IPT_CYC_SAL=0" "IPT_CYC_SAL=1" "IPT_CYC_SAL=0" "IPT_CYC_SAL=1"; do echo "$m" >> gpurun_out/plan_ab.txt; env $m timeout 600 python tools/plan_ab.py >> gpurun_out/plan_ab.txt 2>&1; done
