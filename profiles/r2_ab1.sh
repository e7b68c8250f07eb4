cd $GRAFT_REPO_ROOT
timeout 1200 python -m pytest tests -q -m gpu -x -k "parity or fullsize or multirank or validation" > gpurun_out/pytest_gpu_new.log 2>&1; echo pytest=$?
tail -4 gpurun_out/pytest_gpu_new.log
VARIANTS="r1 new g4 mix" ARGS="--steps 50" bash profiles/ab_run.sh
