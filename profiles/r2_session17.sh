# DRAM traffic of k_fused3 at C5 and C4 (P = 1) with the final kernel; fused sensitivity sweep (final kernel)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2t
timeout 1500 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:k_fused3 -s 2 -c 1 --csv --log-file gpurun_out/r2t/C5_dram.csv python bench.py --config C5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo c5=$?
timeout 1500 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum,l1tex__data_pipe_lsu_wavefronts.avg.pct_of_peak_sustained_elapsed --clock-control none -k regex:k_fused3 -s 2 -c 1 --csv --log-file gpurun_out/r2t/C4_dram.csv python bench.py --config C4 --scaling strong --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo c4=$?
cat gpurun_out/r2t/C5_dram.csv gpurun_out/r2t/C4_dram.csv | grep -v "^==" | cut -c1-300
rm -rf gpurun_out/sweep
VARIANTS=fused bash profiles/sweep_run.sh
python profiles/sweep_table.py gpurun_out/sweep
