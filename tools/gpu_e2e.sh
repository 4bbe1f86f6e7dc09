cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
for s in 2 3 4; do for q in 4 8; do
timeout 300 python bench.py --steps 3 --warmup 3 --no-cpu --autotune 4 --e2e-streams $s --queues $q --e2e-steps 2 2>/dev/null | python -c "
import json,sys; d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('streams $s queues $q', d['value'], d['e2e'])"
done; done
