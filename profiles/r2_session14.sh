# A/B of the attitude gather-copy format: window (default for n_att <= 2^20) vs knot (LSQR_KNOT_GATHER=1)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab14
for rep in 1 2; do
  for z in 0 1; do
    if [ $z = 1 ]; then export LSQR_KNOT_GATHER=1; else unset LSQR_KNOT_GATHER; fi
    timeout 300 python bench.py --config C2 --steps 100 --no-e2e --no-cpu-baseline > gpurun_out/ab14/C2_knot$z.$rep.json 2>/dev/null
    timeout 600 python bench.py --config C3 --steps 50 --no-e2e --no-cpu-baseline > gpurun_out/ab14/C3_knot$z.$rep.json 2>/dev/null
  done
done
unset LSQR_KNOT_GATHER
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ab14/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, "%.4e" % d["value"], d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], d["clocks"]["sm_mhz"], d["api_products"]["aprod1_frac"])
    except Exception as e:
        print(f, "ERR", e)
PY
timeout 1500 python -m pytest tests -q -m gpu -k "parity or multirank or fullsize" > gpurun_out/pytest_s14.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_s14.log
