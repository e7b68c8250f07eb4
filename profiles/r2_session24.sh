# Launch list of the final build (default bench command, short): shares per kernel
cd $GRAFT_REPO_ROOT
mkdir -p gpurun_out/r2g
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv --log-file gpurun_out/r2g/launches_C3.csv python bench.py --steps 8 --warmup 3 --no-e2e --no-cpu-baseline > /dev/null 2>&1; echo ncul=$?
ls -la gpurun_out/r2g
