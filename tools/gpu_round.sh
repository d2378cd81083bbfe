#!/bin/bash
# One gpurun session: build, the named GPU test files (or the whole -m gpu
# suite with ALL=1), optional extra commands from $EXTRA.  Logs: gpurun_out/$TAG_*
cd "$(dirname "$0")/.."
TAG=${TAG:-run}
mkdir -p gpurun_out
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/${TAG}_build.log 2>&1 || { tail -20 gpurun_out/${TAG}_build.log; exit 1; }
if [ -n "$TESTS" ]; then
  timeout ${TTIME:-900} python -m pytest $TESTS -m gpu -q -x > gpurun_out/${TAG}_tests.log 2>&1
  echo "tests rc=$?: $(tail -1 gpurun_out/${TAG}_tests.log)"
fi
if [ -n "$ALL" ]; then
  timeout ${TTIME:-1200} python -m pytest tests -m gpu -q > gpurun_out/${TAG}_all.log 2>&1
  echo "all rc=$?: $(tail -1 gpurun_out/${TAG}_all.log)"
fi
if [ -n "$EXTRA" ]; then
  bash -c "$EXTRA"
fi
