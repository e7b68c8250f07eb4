cd $GRAFT_REPO_ROOT
timeout 900 python tests/tools/sigma_study.py > gpurun_out/sigma_study.txt 2>&1; echo rc=$?
cat gpurun_out/sigma_study.txt | tail -40
