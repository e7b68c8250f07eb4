# Round-2 profiling session: full ncu captures (with source) of the fused kernel at C2 and C3 + launch list.
# Usage (from the repo root, on the GPU box): bash profiles/r2_profile.sh [tag]
cd $GRAFT_REPO_ROOT
TAG=${1:-base}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total --format=csv
timeout 900 ncu --set full --clock-control none --import-source on -k regex:k_fused3 -s 2 -c 1 \
  -o gpurun_out/r2_${TAG}_fused3_C2 -f python bench.py --steps 3 --warmup 3 --no-e2e --no-cpu-baseline \
  > gpurun_out/r2_${TAG}_ncu_C2.log 2>&1; echo ncuC2=$?
timeout 1500 ncu --set full --clock-control none --import-source on -k regex:k_fused3 -s 2 -c 1 \
  -o gpurun_out/r2_${TAG}_fused3_C3 -f python bench.py --config C3 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline \
  > gpurun_out/r2_${TAG}_ncu_C3.log 2>&1; echo ncuC3=$?
timeout 900 python bench.py --config C3 --steps 20 --no-e2e --no-cpu-baseline > gpurun_out/r2_${TAG}_bench_C3.json 2> gpurun_out/r2_${TAG}_bench_C3.err; echo benchC3=$?
timeout 600 python bench.py --steps 100 --no-e2e --no-cpu-baseline > gpurun_out/r2_${TAG}_bench_C2.json 2> gpurun_out/r2_${TAG}_bench_C2.err; echo benchC2=$?
cut -c1-300 gpurun_out/r2_${TAG}_bench_C3.json gpurun_out/r2_${TAG}_bench_C2.json
