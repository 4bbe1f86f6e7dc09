cd $GRAFT_REPO_ROOT
export CASES="[('S128',(1,4000,1500,32)),('S256',(1,12000,250,64)),('S480',(1,7200,150,120)),('S512',(1,12800,117,128))]"
KNOBS='[{}, {"IPT_CYC_G":"1","IPT_CYC_R":"8"}, {"IPT_CYC_G":"2","IPT_CYC_R":"4"}, {"IPT_CYC_G":"2","IPT_CYC_R":"8"}, {"IPT_CYC_G":"4","IPT_CYC_R":"8"}, {"IPT_CYC_G":"4","IPT_CYC_R":"2"}, {"IPT_CYC_G":"8","IPT_CYC_R":"8"}, {"IPT_CYC_G":"8","IPT_CYC_R":"4"}]' timeout 900 python tools/cyc_knobs.py > gpurun_out/cyc_knobs.log 2>&1
