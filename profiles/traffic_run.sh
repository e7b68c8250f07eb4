# DRAM bytes per launch of the dominant kernels at the large configurations (ncu, 2 metrics) -> gpurun_out/traffic/
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/traffic
M=dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum
timeout 900 ncu --metrics $M --clock-control none -k regex:k_fused3 -s 2 -c 1 --csv --log-file gpurun_out/traffic/C3_fused.csv python bench.py --config C3 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo c3f=$?
timeout 900 ncu --metrics $M --clock-control none -k regex:"k_aprod1|k_fused3" -s 4 -c 2 --csv --log-file gpurun_out/traffic/C3_twopass.csv python bench.py --config C3 --two-pass --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo c3t=$?
timeout 1500 ncu --metrics $M --clock-control none -k regex:k_fused3 -s 2 -c 1 --csv --log-file gpurun_out/traffic/C5_fused.csv python bench.py --config C5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo c5f=$?
grep -h "dram__\|gpu__time" gpurun_out/traffic/*.csv | cut -c1-250
