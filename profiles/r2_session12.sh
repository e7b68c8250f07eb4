# A/B of the attitude window accumulator z4 (LSQR_NO_Z4=1 disables it), then the parity subset with it
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab12
for rep in 1 2; do
  for z in 0 1; do
    if [ $z = 1 ]; then export LSQR_NO_Z4=1; else unset LSQR_NO_Z4; fi
    timeout 300 python bench.py --config C2 --steps 100 --no-e2e --no-cpu-baseline > gpurun_out/ab12/C2_noz4$z.$rep.json 2>/dev/null
    timeout 600 python bench.py --config C3 --steps 50 --no-e2e --no-cpu-baseline > gpurun_out/ab12/C3_noz4$z.$rep.json 2>/dev/null
  done
done
unset LSQR_NO_Z4
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ab12/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, "%.4e" % d["value"], d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], d["clocks"]["sm_mhz"], d["gpu_launches"])
    except Exception as e:
        print(f, "ERR", e)
PY
timeout 1500 python -m pytest tests -q -m gpu -k "parity or multirank or repro or validation or bench" > gpurun_out/pytest_s12.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_s12.log
