# Round-end check of the committed state: GPU tests, smoke, default bench line (C3)
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/final
timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/final/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/final/pytest_gpu.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
S=$(date +%s); timeout 1500 python bench.py > gpurun_out/final/bench.json 2> gpurun_out/final/bench.err; echo bench=$? $(( $(date +%s) - S ))s
cut -c1-400 gpurun_out/final/bench.json
