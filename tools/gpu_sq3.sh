cd $GRAFT_REPO_ROOT; mkdir -p gpurun_out
timeout 300 python -m pytest tests -m gpu -q -x -k "square_swap_sides" -p no:cacheprovider > gpurun_out/pytest_sq.log 2>&1; echo "rc=$?" >> gpurun_out/pytest_sq.log
export SHAPES='[(16384,4),(20000,4),(8192,4),(1024,4)]'
export VARIANTS='[{},{"IPT_SQ_TB":384},{"IPT_SQ_NT":1024},{},{"IPT_SQ_TB":384},{"IPT_SQ_NT":1024}]'
timeout 900 python tools/sq_sweep.py > gpurun_out/sq_sweep.txt 2>&1
IPT_SQ_TB=384 IPT_SQ_FORCE=1 timeout 120 python -c "
import torch, paper_conf_ppopp_sunggggh14_b200 as ipt
for g in (100, 96, 1000, 2049):
    t=torch.randint(0,1<<30,(3*g*g,),dtype=torch.int32,device='cuda'); r=t.view(3,g,g).transpose(1,2).contiguous().view(-1)
    ipt.ipt_010_(t,3,g,g); print(g, torch.equal(t,r))
" >> gpurun_out/sq_sweep.txt 2>&1
