cd $GRAFT_REPO_ROOT
timeout 1500 python bench.py > gpurun_out/bench_default_r2c.json 2> gpurun_out/bench_default_r2c.err; echo bench=$?
tail -3 gpurun_out/bench_default_r2c.err
cut -c1-300 gpurun_out/bench_default_r2c.json
timeout 1500 python -m pytest tests -q -m gpu -k "test_gpu_parity" > gpurun_out/pytest_gpu_parity_r2c.log 2>&1; echo pytest=$?
tail -25 gpurun_out/pytest_gpu_parity_r2c.log
