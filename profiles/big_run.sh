# Large-configuration bench lines (C3, C5 per GPU, C4 at P = 1) on one B200; outputs under gpurun_out/big/
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/big
timeout 900 python bench.py --config C3 --no-cpu-baseline --no-e2e > gpurun_out/big/bench_C3_fused.json 2> gpurun_out/big/C3.err; echo C3=$?
timeout 1200 python bench.py --config C5 --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/big/bench_C5_fused.json 2> gpurun_out/big/C5.err; echo C5=$?
timeout 1200 python bench.py --config C5 --two-pass --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/big/bench_C5_twopass.json 2> gpurun_out/big/C5t.err; echo C5t=$?
timeout 1500 python bench.py --config C4 --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/big/bench_C4_fused.json 2> gpurun_out/big/C4.err; echo C4=$?
for f in gpurun_out/big/*.json; do echo $f; cut -c1-200 $f; done
tail -3 gpurun_out/big/*.err
