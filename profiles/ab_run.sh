# A/B of experiment builds under .variants/<name> (bench lines only; outputs under gpurun_out/ab/)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab
for rep in 1 2; do for v in $VARIANTS; do
  (cd .variants/$v && timeout 300 python bench.py --no-e2e --no-cpu-baseline $ARGS > ../../gpurun_out/ab/${v}_C2_$rep.json 2>/dev/null)
done; done
for v in $VARIANTS; do
  (cd .variants/$v && timeout 600 python bench.py --config C3 --no-e2e --no-cpu-baseline $ARGS > ../../gpurun_out/ab/${v}_C3.json 2>/dev/null)
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ab/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, "%.4e" % d["value"], d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], d["clocks"]["sm_mhz"])
    except Exception as e:
        print(f, "ERR", e)
PY
