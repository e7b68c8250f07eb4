# GPU tests of one experiment build (TESTDIR, default the repo) + A/B bench lines of VARIANTS
cd $GRAFT_REPO_ROOT
(cd ${TESTDIR:-.} && timeout 1500 python -m pytest tests -x -q -m gpu > $GRAFT_REPO_ROOT/gpurun_out/pytest_gpu.log 2>&1; echo pytest=$?)
tail -3 gpurun_out/pytest_gpu.log
bash profiles/ab_run.sh
