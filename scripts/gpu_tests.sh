#!/bin/bash
# GPU tests only, fail fast, verbose.  Usage: bash scripts/gpu_tests.sh TAG [pytest args...]
TAG=${1:-t}; shift
OUT=gpurun_out/$TAG
mkdir -p $OUT
export PYTHONUNBUFFERED=1
timeout ${GPU_TEST_TIMEOUT:-900} python -m pytest -m gpu -x -v -rA --timeout 300 -p no:cacheprovider "$@" > $OUT/pytest.txt 2>&1
echo "pytest rc=$?" >> $OUT/pytest.txt
grep -E "PASSED|FAILED|ERROR|rc=" $OUT/pytest.txt | tail -40
