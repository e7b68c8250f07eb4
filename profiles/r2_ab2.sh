cd $GRAFT_REPO_ROOT
free -g | head -2; nproc; grep "model name" /proc/cpuinfo | head -1
timeout 1200 python -m pytest tests -q -m gpu -x -k "parity or fullsize or multirank" > gpurun_out/pytest_gpu_g4.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu_g4.log
VARIANTS="r1 g4" ARGS="--steps 50" bash profiles/ab_run.sh
/usr/bin/time -v timeout 1500 python bench.py > gpurun_out/bench_default_g4.json 2> gpurun_out/bench_default_g4.err; echo bench=$?
tail -25 gpurun_out/bench_default_g4.err | grep -E "Maximum resident|Elapsed|Error|error" 
cut -c1-600 gpurun_out/bench_default_g4.json
