cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python bench.py --steps 10 --warmup 3 --no-cpu --no-e2e ${BENCH_ARGS} > gpurun_out/bench.json 2>gpurun_out/bench.err
python -c "
import json; d=json.loads(open('gpurun_out/bench.json').read().strip().splitlines()[-1]); print(d['value'], d['hbm_frac_stage_scaled'], d['roofline']['kernel'], d['roofline']['frac'], d['roofline']['per_kernel_ms'])
for k,v in d['per_shape'].items(): print(k, d['config']['plans'][k]['m'], d['config']['plans'][k]['n'], v)"
