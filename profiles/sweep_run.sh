# SURVEY §8(d) sensitivity sweep on the C3 shape (208 M rows): n_att x n_instr, fused and two-pass iterations.
# Outputs one bench line per point under gpurun_out/sweep/.  ATTS / INSTRS / VARIANTS override the grid.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/sweep
for na in ${ATTS:-1200 30000 300000 3000000}; do for ni in ${INSTRS:-60 6000 60000}; do for v in ${VARIANTS:-fused two-pass}; do
  timeout 600 python bench.py --config C3 --n-att $na --n-instr $ni --$v --steps 20 --warmup 3 --no-e2e \
    --no-cpu-baseline > gpurun_out/sweep/att${na}_instr${ni}_${v}.json 2> gpurun_out/sweep/att${na}_instr${ni}_${v}.err
  echo "$na $ni $v rc=$?"
done; done; done
