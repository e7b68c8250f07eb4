# GPU test session: pytest -m gpu (full), smoke.  Usage: bash profiles/gpu_tests.sh [tag] [pytest -k expr]
cd $GRAFT_REPO_ROOT
TAG=${1:-r2}
K=${2:-}
if [ -n "$K" ]; then
  timeout 2400 python -m pytest tests -q -m gpu -k "$K" -x > gpurun_out/pytest_gpu_${TAG}.log 2>&1; echo pytest=$?
else
  timeout 2400 python -m pytest tests -q -m gpu > gpurun_out/pytest_gpu_${TAG}.log 2>&1; echo pytest=$?
fi
tail -15 gpurun_out/pytest_gpu_${TAG}.log
timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -1
