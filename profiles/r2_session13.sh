# C5 / C4 with the attitude window accumulator forced on (n_att = 3e6: 96 MB) vs the default (off)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab13
for rep in 1 2; do
  timeout 900 python bench.py --config C5 --steps 20 --no-e2e --no-cpu-baseline > gpurun_out/ab13/C5_default.$rep.json 2>/dev/null
  (cd .variants/z4big && timeout 900 python bench.py --config C5 --steps 20 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab13/C5_z4.$rep.json 2>/dev/null)
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ab13/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, "%.4e" % d["value"], d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], d["clocks"]["sm_mhz"])
    except Exception as e:
        print(f, "ERR", e)
PY
