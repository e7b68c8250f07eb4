# Experiment build (-DLSQR_WARP_TIMING=4): per-warp start/finish times of the 5th k_fused3 launch at C3 and C2
cd $GRAFT_REPO_ROOT/.variants/wt
mkdir -p ../../gpurun_out/ab27
for cfg in C3 C2; do
timeout 600 python -c "
import workloads as W, paper_conf_sc_malenzacsbvba24_b200 as avu
s = avu.Solver.synthetic(W.$cfg)
s.precondition()
out = s.solve(itn_limit=8, atol=0, btol=0, conlim=0, fixed_count=True, fused=True)
print('itn', out['itn'])
" > ../../gpurun_out/ab27/wt_$cfg.txt 2>&1; echo $cfg=$? $(grep -c '^WT' ../../gpurun_out/ab27/wt_$cfg.txt)
done
