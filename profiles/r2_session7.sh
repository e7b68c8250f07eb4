# Round-2 measurement session: full GPU suite, smoke, bench lines (C3 default, C2, two-pass, C4 strong T(1), C5,
# reference arm), ncu launch list and full captures of k_fused3.  Outputs under gpurun_out/r2/.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total,power.limit --format=csv
S=$(date +%s); timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/r2/pytest_gpu.log 2>&1; echo pytest=$? $(( $(date +%s) - S ))s
tail -4 gpurun_out/r2/pytest_gpu.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2/smoke.log 2>&1; tail -1 gpurun_out/r2/smoke.log
S=$(date +%s); timeout 1500 python bench.py > gpurun_out/r2/bench_C3_default.json 2> gpurun_out/r2/bench_C3_default.err; echo bench=$? $(( $(date +%s) - S ))s
timeout 900 python bench.py --config C2 > gpurun_out/r2/bench_C2.json 2> gpurun_out/r2/bench_C2.err; echo benchC2=$?
timeout 900 python bench.py --two-pass --no-e2e --no-cpu-baseline > gpurun_out/r2/bench_C3_twopass.json 2>/dev/null; echo twopass=$?
timeout 1200 python bench.py --config C4 --scaling strong --steps 20 --no-e2e --no-cpu-baseline > gpurun_out/r2/bench_C4_strong_P1.json 2>/dev/null; echo C4=$?
timeout 1200 python bench.py --config C5 --steps 20 --no-e2e --no-cpu-baseline > gpurun_out/r2/bench_C5.json 2>/dev/null; echo C5=$?
S=$(date +%s); timeout 900 python bench.py --impl reference > gpurun_out/r2/bench_reference.json 2> gpurun_out/r2/bench_reference.err; echo ref=$? $(( $(date +%s) - S ))s
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2/launches_C3.csv python bench.py --steps 8 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncul=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fused3 -s 2 -c 1 -o gpurun_out/r2/full_fused3_C3 -f python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncuC3=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fused3 -s 2 -c 1 -o gpurun_out/r2/full_fused3_C2 -f python bench.py --config C2 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncuC2=$?
for f in gpurun_out/r2/bench_*.json; do echo $f; cut -c1-200 $f; done
