cd $GRAFT_REPO_ROOT
KNOBS='[{}, {"IPT_CYC_SCRAMBLE":"2"}, {"IPT_CYC_SCRAMBLE":"0"}, {"IPT_CYC_SCRAMBLE":"2", "IPT_CYC_FENCE":"0"}]' timeout 900 python tools/cyc_knobs.py > gpurun_out/cyc_knobs.log 2>&1
