# A/B of the window accumulator layout: z4[k0][a][j] (default) vs z4[a][k0][j] (LSQR_Z4_AXIS_OUTER=1)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab15
for rep in 1 2; do
  for z in 0 1; do
    if [ $z = 1 ]; then export LSQR_Z4_AXIS_OUTER=1; else unset LSQR_Z4_AXIS_OUTER; fi
    timeout 300 python bench.py --config C2 --steps 100 --no-e2e --no-cpu-baseline > gpurun_out/ab15/C2_axouter$z.$rep.json 2>/dev/null
    timeout 600 python bench.py --config C3 --steps 50 --no-e2e --no-cpu-baseline > gpurun_out/ab15/C3_axouter$z.$rep.json 2>/dev/null
  done
done
unset LSQR_Z4_AXIS_OUTER
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ab15/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, "%.4e" % d["value"], d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], d["clocks"]["sm_mhz"], d["api_products"]["aprod1_frac"])
    except Exception as e:
        print(f, "ERR", e)
PY
timeout 1500 python -m pytest tests -q -m gpu -k "parity or multirank or fullsize" > gpurun_out/pytest_s14.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_s14.log
