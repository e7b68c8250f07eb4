# GPU tests, then the IG + shared-memory-attitude sweep points -> gpurun_out/
cd $GRAFT_REPO_ROOT
timeout 1500 python -m pytest tests -x -q -m gpu > gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?
tail -3 gpurun_out/pytest_gpu.log
ATTS="1200 3000" INSTRS="60000" bash profiles/sweep_run.sh
