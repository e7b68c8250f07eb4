# Experiment builds (-DLSQR_WARP_TIMING=N): per-warp start/finish times (globaltimer) of the N-th k_fused3 launch
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab28
for v in wt wt20; do for cfg in C3 C2; do
(cd .variants/$v && timeout 600 python -c "
import ctypes, numpy as np, workloads as W, paper_conf_sc_malenzacsbvba24_b200 as avu
from paper_conf_sc_malenzacsbvba24_b200 import _capi
s = avu.Solver.synthetic(W.$cfg)
s.precondition()
out = s.solve(itn_limit=24, atol=0, btol=0, conlim=0, fixed_count=True, fused=True)
buf = np.zeros(2 * 148 * 16, dtype=np.uint64)
rc = _capi.lib().lsqr_debug_warp_times(ctypes.c_void_p(buf.ctypes.data))
np.save('../../gpurun_out/ab28/${v}_$cfg.npy', buf)
print('rc', rc, 'itn', out['itn'])
"); echo $v $cfg $?
done; done
