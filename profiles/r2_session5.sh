cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab5
for rep in 1 2 3; do for v in base noidx not5 new; do
  (cd .variants/$v && timeout 300 python bench.py --config C2 --steps 100 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab5/${v}_C2_$rep.json 2>/dev/null)
done; done
for v in base new; do
  (cd .variants/$v && timeout 600 python bench.py --config C3 --steps 30 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab5/${v}_C3.json 2>/dev/null)
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ab5/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, "%.4e" % d["value"], d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], d["clocks"]["sm_mhz"])
    except Exception as e:
        print(f, "ERR", e)
PY
timeout 1800 python -m pytest tests -q -m gpu -k "sigma or validation or bench or parity" > gpurun_out/pytest_gpu_s5.log 2>&1; echo pytest=$?
tail -6 gpurun_out/pytest_gpu_s5.log
grep -E "^validation|se at k" gpurun_out/pytest_gpu_s5.log | head -30
