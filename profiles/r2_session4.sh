# Session 4: the oracle's C3 reference for NEXT-3 (background, CPU), meanwhile the full GPU suite, the fused
# kernel's time breakdown at C3 (experiment build), and a full ncu capture of k_fused3 at C3.
cd $GRAFT_REPO_ROOT
(python -m tests.golden.make_next3 C3 > gpurun_out/make_next3_C3.log 2>&1; cp tests/golden/next3_C3.npz gpurun_out/ 2>/dev/null) &
BG=$!
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu_s4.log 2>&1; echo pytest=$?
tail -12 gpurun_out/pytest_gpu_s4.log
mkdir -p gpurun_out/diag
for d in 0 1 2 4 8 16 31; do
  (cd .variants/diag && LSQR_DIAG=$d timeout 600 python bench.py --config C3 --steps 20 --no-e2e --no-cpu-baseline > ../../gpurun_out/diag/C3_$d.json 2>/dev/null)
done
python - <<'PY'
import json
for d in (0, 1, 2, 4, 8, 16, 31):
    try:
        j = json.load(open(f"gpurun_out/diag/C3_{d}.json"))
        print("diag", d, j["roofline"]["avg_launch_ms"], j["clocks"]["sm_mhz"])
    except Exception as e:
        print("diag", d, "ERR", e)
PY
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:k_fused3 -s 2 -c 1 -o gpurun_out/r2_g4_fused3_C3 -f python bench.py --config C3 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/r2_g4_ncu_C3.log 2>&1; echo ncu=$?
wait $BG
tail -2 gpurun_out/make_next3_C3.log
ls -la gpurun_out/next3_C3.npz
