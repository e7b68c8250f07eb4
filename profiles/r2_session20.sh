# k_post folds the z4 window accumulator (P = 1): full GPU suite, smoke, default C3 line, C2 line
cd $GRAFT_REPO_ROOT
bash profiles/final_check.sh
timeout 600 python bench.py --config C2 --steps 100 > gpurun_out/final/bench_C2.json 2>/dev/null; echo c2=$?
cut -c1-300 gpurun_out/final/bench_C2.json
