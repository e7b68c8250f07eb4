# Final state: GPU suite, smoke, default C3 line, reference arm (N = 1)
cd $GRAFT_REPO_ROOT
bash profiles/final_check.sh
S=$(date +%s); timeout 1200 python bench.py --impl reference > gpurun_out/final/bench_reference.json 2> gpurun_out/final/bench_reference.err; echo ref=$? $(( $(date +%s) - S ))s
cut -c1-600 gpurun_out/final/bench_reference.json
