# A/B of experiment builds (.variants/<name>) at C3 and C5 (bench lines) + ncu DRAM bytes of k_fused3 at C5
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/ab
for rep in 1 2; do for v in $VARIANTS; do
  (cd .variants/$v && timeout 900 python bench.py --config C3 --steps 20 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab/${v}_C3_$rep.json 2>/dev/null)
  (cd .variants/$v && timeout 1200 python bench.py --config C5 --steps 20 --no-e2e --no-cpu-baseline > ../../gpurun_out/ab/${v}_C5_$rep.json 2>/dev/null)
done; done
for v in $VARIANTS; do
  (cd .variants/$v && timeout 1500 ncu --metrics dram__bytes_read.sum,dram__bytes_write.sum,gpu__time_duration.sum --clock-control none -k regex:k_fused3 -s 2 -c 1 --csv --log-file ../../gpurun_out/ab/${v}_C5_dram.csv python bench.py --config C5 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1)
done
python - <<'PY'
import json, glob
for f in sorted(glob.glob("gpurun_out/ab/*.json")):
    try:
        d = json.loads(open(f).read().strip().splitlines()[-1])
        print(f, "%.4e" % d["value"], d["roofline"]["avg_launch_ms"], d["roofline"]["frac"], d["clocks"]["sm_mhz"], d["repetitions"]["ms_per_step"])
    except Exception as e:
        print(f, "ERR", e)
PY
