cd $GRAFT_REPO_ROOT
timeout 1800 python -m pytest tests -q -m gpu -k "parity or multirank or fullsize" > gpurun_out/pytest_s10.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_s10.log
timeout 900 python bench.py --two-pass --no-e2e --no-cpu-baseline > gpurun_out/bench_C3_twopass_g4.json 2>/dev/null; echo twopass=$?
python -c "
import json; d=json.load(open('gpurun_out/bench_C3_twopass_g4.json'))
print(d['value'], d['iteration_roofline'], d['api_products'], d['clocks'])"
