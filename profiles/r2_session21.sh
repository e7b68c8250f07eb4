# A/B: z4 fold in k_post (P = 1) vs the separate k_att_fold launch (C2); shared-memory slot-layout microbenchmark
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab21
./microbench/mb_slot | tee gpurun_out/ab21/mb_slot.txt
for rep in 1 2 3; do for v in base fold; do
  (cd .variants/$v && timeout 300 python bench.py --config C2 --steps 200 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab21/${v}_C2_$rep.json 2>/dev/null)
done; done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ab21/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, "%.4e" % d["value"], d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], d["clocks"]["sm_mhz"])
    except Exception as e:
        print(f, "ERR", e)
PY
