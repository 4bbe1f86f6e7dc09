cd $GRAFT_REPO_ROOT
KNOBS_FILE=tools/knobs.txt CASES_FILE=tools/cases.txt timeout 900 python tools/cyc_knobs.py > gpurun_out/knobs.txt 2>&1
