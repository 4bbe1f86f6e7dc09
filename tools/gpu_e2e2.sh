cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for cfg in "2 4" "4 4" "4 2" "4 3" "6 2" "6 3"; do set -- $cfg
  timeout 600 python bench.py --steps 3 --warmup 3 --no-cpu --e2e-steps $1 --e2e-streams $2 > gpurun_out/e2e_$1_$2.json 2>>gpurun_out/e2e.err
done
