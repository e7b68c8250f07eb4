# Final round-2 measurement of the committed kernel: bench lines (C3 default, C2, C3 two-pass, C4 P=1, C5, reference
# arm), ncu launch list + full captures (C2, C3), full GPU suite.  Outputs under gpurun_out/r2f/.
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2f
S=$(date +%s); timeout 1500 python bench.py > gpurun_out/r2f/bench_C3_default.json 2> gpurun_out/r2f/bench_C3_default.err; echo bench=$? $(( $(date +%s) - S ))s
timeout 900 python bench.py --config C2 > gpurun_out/r2f/bench_C2.json 2> /dev/null; echo benchC2=$?
timeout 900 python bench.py --two-pass --no-e2e --no-cpu-baseline > gpurun_out/r2f/bench_C3_twopass.json 2>/dev/null; echo twopass=$?
timeout 1200 python bench.py --config C4 --scaling strong --steps 20 --no-e2e --no-cpu-baseline > gpurun_out/r2f/bench_C4_strong_P1.json 2>/dev/null; echo C4=$?
timeout 1200 python bench.py --config C5 --steps 20 --no-e2e --no-cpu-baseline > gpurun_out/r2f/bench_C5.json 2>/dev/null; echo C5=$?
timeout 900 python bench.py --impl reference > gpurun_out/r2f/bench_reference.json 2>/dev/null; echo ref=$?
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2f/launches_C3.csv python bench.py --steps 8 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncul=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fused3 -s 2 -c 1 -o gpurun_out/r2f/full_fused3_C3 -f python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncuC3=$?
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fused3 -s 2 -c 1 -o gpurun_out/r2f/full_fused3_C2 -f python bench.py --config C2 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncuC2=$?
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/r2f/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/r2f/pytest_gpu.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/r2f/smoke.log 2>&1; tail -1 gpurun_out/r2f/smoke.log
for f in gpurun_out/r2f/bench_*.json; do echo $f; cut -c1-160 $f; done
