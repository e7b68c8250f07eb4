# A/B: leftover-piece granularity of k_fused3's dynamic balance (C3), against HEAD
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab30
run() { (cd .variants/$1 && env $3 timeout 600 python bench.py --config C3 --steps 50 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab30/$2.json 2>/dev/null); }
for rep in 1 2; do
  run base base_$rep ""
  run dyn np4_$rep "LSQR_DYN_NP=4"
  run dyn np8_$rep "LSQR_DYN_NP=8"
  run dyn np16_$rep "LSQR_DYN_NP=16"
  run dyn f05np8_$rep "LSQR_DYN_FRAC=0.05 LSQR_DYN_NP=8"
  run dyn f12np16_$rep "LSQR_DYN_FRAC=0.12 LSQR_DYN_NP=16"
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ab30/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        ms, mhz = d["roofline"]["avg_launch_ms"], d["clocks"]["sm_mhz"]
        print(f, "%.4e" % d["value"], ms, d["roofline"]["frac"], mhz, "ms*GHz %.2f" % (ms * mhz / 1000))
    except Exception as e:
        print(f, "ERR", e)
PY
