# A/B: k_fused3 with leftover pieces taken dynamically (dyn; LSQR_DYN_FRAC = 0: static only) vs HEAD (base); parity
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab29
(cd .variants/dyn && timeout 900 python -m pytest tests -q -m gpu -x -k "test_lsqr_C2_full or edge_cases or layouts or tiny or teacher_forced_step_C2 or free_run or aprod_full" 2>&1 | tail -3)
for rep in 1 2; do
  for v in base dyn; do
    (cd .variants/$v && timeout 300 python bench.py --config C2 --steps 200 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab29/${v}_C2_$rep.json 2>/dev/null)
    (cd .variants/$v && timeout 600 python bench.py --config C3 --steps 50 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab29/${v}_C3_$rep.json 2>/dev/null)
  done
  (cd .variants/dyn && LSQR_DYN_FRAC=0 timeout 600 python bench.py --config C3 --steps 50 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab29/dyn0_C3_$rep.json 2>/dev/null)
  (cd .variants/dyn && LSQR_DYN_FRAC=0.15 timeout 600 python bench.py --config C3 --steps 50 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab29/dyn15_C3_$rep.json 2>/dev/null)
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ab29/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, "%.4e" % d["value"], d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], d["clocks"]["sm_mhz"])
    except Exception as e:
        print(f, "ERR", e)
PY
