# DRAM bytes of k_fused3 at C5 with parts of the shared-slice work removed (experiment build, results wrong by design)
cd $GRAFT_REPO_ROOT/.variants/diag
mkdir -p ../../gpurun_out/diag
for m in 0 2 4 1; do
  LSQR_DIAG=$m timeout 1500 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_fused3 -s 2 -c 1 --csv --log-file ../../gpurun_out/diag/C5_diag$m.csv python bench.py --config C5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo m$m=$?
done
