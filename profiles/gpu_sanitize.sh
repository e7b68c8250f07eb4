cd $GRAFT_REPO_ROOT
timeout 2400 python -m pytest tests/test_sanitizer.py -x -q -m gpu > gpurun_out/pytest_san.log 2>&1; echo san=$?
tail -5 gpurun_out/pytest_san.log
