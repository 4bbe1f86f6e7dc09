cd $GRAFT_REPO_ROOT
KNOBS='[{}, {"IPT_CYC_IDX64":"1"}, {"IPT_CYC_FENCE":"0"}, {"IPT_CYC_G":"8","IPT_CYC_R":"4"}, {"IPT_CYC_G":"16","IPT_CYC_R":"2"}, {"IPT_CYC_G":"8","IPT_CYC_R":"2"}]' timeout 900 python tools/cyc_knobs.py > gpurun_out/cyc_knobs.log 2>&1
timeout 900 python -m pytest tests/test_gpu_parity.py -q -x --timeout 300 -p no:cacheprovider > gpurun_out/pytest_gpu.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_gpu.log
