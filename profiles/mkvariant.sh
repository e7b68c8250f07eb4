# Experiment build: copy of the working tree (or of a git revision) under .variants/<name>, library built with extra
# nvcc flags.  Usage: bash profiles/mkvariant.sh <name> "<nvcc flags>" [git-rev]
set -e
cd "$(dirname "$0")/.."
NAME=$1; FLAGS=$2; REV=$3
rm -rf .variants/$NAME && mkdir -p .variants/$NAME
if [ -n "$REV" ]; then
  git archive "$REV" | tar -x -C .variants/$NAME
else
  tar --exclude=.git --exclude=.variants --exclude=gpurun_out --exclude='*.so' -cf - . | tar -x -C .variants/$NAME
fi
(cd .variants/$NAME && LSQR_NVCC_EXTRA="$FLAGS" python -c "
from paper_conf_sc_malenzacsbvba24_b200 import build as b; b.build(force=True)
import oracle; oracle.build(force=True)" > /dev/null)
echo built .variants/$NAME
