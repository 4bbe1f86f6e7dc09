cd $GRAFT_REPO_ROOT
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x --timeout 300 -p no:cacheprovider -k "100 or transpose or stress" > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
export CASES="[('S128',(1,4000,1500,32)),('S256',(1,12000,250,64)),('S480',(1,7200,150,120)),('S512',(1,12800,117,128)),('S640_st3',(75,50,320,160)),('S1024',(1,12000,16,256)),('S1600_st1',(1,9600,50,400))]"
KNOBS='[{"IPT_CYC_FASTLOOP":"0"}, {"IPT_CYC_FASTLOOP":"1"}]' timeout 900 python tools/cyc_knobs.py > gpurun_out/cyc_knobs.log 2>&1
