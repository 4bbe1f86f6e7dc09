cd $GRAFT_REPO_ROOT
for cfg in "IPT_CYC_PF=0" "IPT_CYC_PF=1" "IPT_CYC_PF=2" "IPT_CYC_PF=3" "IPT_CYC_PF=2 IPT_CYC_FENCE=0"; do
  env $cfg CFG="$cfg" timeout 300 python tools/cyc_sweep.py
done > gpurun_out/cyc_sweep.log 2>&1
