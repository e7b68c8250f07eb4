# One gpurun session: GPU tests, bench lines, ncu launch list + full capture (outputs under gpurun_out/).
set -x
cd $GRAFT_REPO_ROOT
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_C2.json 2> gpurun_out/bench_C2.err; echo bench=$?
timeout 600 python bench.py --two-pass --no-cpu-baseline --no-e2e > gpurun_out/bench_C2_twopass.json 2> gpurun_out/bench_C2_twopass.err; echo bench2=$?
timeout 900 python bench.py --config C3 --two-pass --no-cpu-baseline --no-e2e > gpurun_out/bench_C3_twopass.json 2> gpurun_out/bench_C3_twopass.err; echo bench3=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fused3 -s 2 -c 2 -o gpurun_out/full_lean2_C2 -f python bench.py --two-pass --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_f.log 2>&1; echo ncuf=$?
timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/launches_C2_twopass.csv python bench.py --two-pass --steps 8 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/ncu_l.log 2>&1; echo ncul=$?
cat gpurun_out/*.json | cut -c1-300
