# C5 shape (625 M rows) with the attitude slice varied: per-row cost of the shared slice vs working-set size
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/c5natt
for na in 300000 1500000 3000000; do
  timeout 1200 python bench.py --config C5 --n-att $na --steps 20 --warmup 3 --no-e2e --no-cpu-baseline > gpurun_out/c5natt/C5_att$na.json 2>/dev/null; echo $na rc=$?
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/c5natt/*.json")):
    d = json.loads(open(f).read().strip().splitlines()[-1])
    print(f, "%.4e" % d["value"], d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], d["clocks"]["sm_mhz"])
PY
