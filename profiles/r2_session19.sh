# A/B: 4-stage ring, 3-stage ring, 3-stage ring + row-parity z_instr copies (C2, C3), parity of the zpar3 build
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab19
for rep in 1 2; do for v in st4 st3 zpar3; do
  (cd .variants/$v && timeout 300 python bench.py --config C2 --steps 100 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab19/${v}_C2_$rep.json 2>/dev/null)
  (cd .variants/$v && timeout 600 python bench.py --config C3 --steps 50 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab19/${v}_C3_$rep.json 2>/dev/null)
done; done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ab19/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, "%.4e" % d["value"], d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], d["clocks"]["sm_mhz"])
    except Exception as e:
        print(f, "ERR", e)
PY
(cd .variants/zpar3 && timeout 900 python -m pytest tests -q -m gpu -k "test_lsqr_C2_full or edge_cases or layouts" 2>&1 | tail -2)
