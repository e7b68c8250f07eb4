cd $GRAFT_REPO_ROOT
VARIANTS=fused bash profiles/sweep_run.sh
python profiles/sweep_table.py gpurun_out/sweep
timeout 900 python bench.py --force-collectives --steps 50 --no-e2e --no-cpu-baseline > gpurun_out/bench_C3_forced.json 2>/dev/null; echo forced=$?
cut -c1-250 gpurun_out/bench_C3_forced.json
