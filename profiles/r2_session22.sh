# A/B: bank-grouped instrumental slots (default) vs identity slots (LSQR_NO_INSTR_PERM=1), C2 and C3, same box
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab22
for rep in 1 2; do for v in grouped identity; do
  if [ $v = identity ]; then export LSQR_NO_INSTR_PERM=1; else unset LSQR_NO_INSTR_PERM; fi
  timeout 300 python bench.py --config C2 --steps 200 --no-e2e --no-cpu-baseline > gpurun_out/ab22/${v}_C2_$rep.json 2>/dev/null
  timeout 600 python bench.py --config C3 --steps 50 --no-e2e --no-cpu-baseline > gpurun_out/ab22/${v}_C3_$rep.json 2>/dev/null
done; done
unset LSQR_NO_INSTR_PERM
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ab22/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, "%.4e" % d["value"], d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], d["clocks"]["sm_mhz"])
    except Exception as e:
        print(f, "ERR", e)
PY
LSQR_NO_INSTR_PERM=1 timeout 900 python -m pytest tests -q -m gpu -k "test_lsqr_C2_full or edge_cases or layouts" 2>&1 | tail -2
