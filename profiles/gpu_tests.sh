# GPU test suite + default bench line (with api_products) + C3 bench
cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
timeout 600 python bench.py > gpurun_out/bench_C2.json 2> gpurun_out/bench_C2.err; echo bench=$?
timeout 900 python bench.py --config C3 --no-cpu-baseline --no-e2e > gpurun_out/bench_C3.json 2> gpurun_out/bench_C3.err; echo bench3=$?
python -c "
import json
for f in ['gpurun_out/bench_C2.json','gpurun_out/bench_C3.json']:
    d=json.loads(open(f).read().strip().splitlines()[-1]); print(f, d['value'], d['roofline']['frac'], d.get('api_products'), (d.get('cpu_baseline') or {}).get('value'))
"
