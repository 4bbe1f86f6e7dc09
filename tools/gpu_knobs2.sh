cd $GRAFT_REPO_ROOT
export CASES="[('S480_st1',(1,7200,150,120)),('S640_st3',(75,50,320,160)),('S576_st1',(1,7200,125,144)),('S1600_st1',(1,9600,50,400)),('S960_st1',(1,7200,75,240))]"
KNOBS='[{}, {"IPT_CYC_G":"16","IPT_CYC_R":"4"}, {"IPT_CYC_G":"8","IPT_CYC_R":"4"}, {"IPT_CYC_FENCE":"0"}, {"IPT_CYC_REFRESH":"0"}, {"IPT_CYC_SCRAMBLE":"1"}]' timeout 900 python tools/cyc_knobs.py > gpurun_out/cyc_knobs.log 2>&1
