cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x -k "host" -p no:cacheprovider > gpurun_out/pytest_pipe.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_pipe.log
for api in pipeline async pipeline async; do timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --e2e-api $api > gpurun_out/e2e_$api.json 2>>gpurun_out/bench.err; cat gpurun_out/e2e_$api.json >> gpurun_out/e2e_all.txt; done
