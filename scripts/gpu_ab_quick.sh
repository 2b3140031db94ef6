#!/bin/bash
# Product-build A/B check: the variant-5 parity subset, then bench lines for several T.
TAG=${1:-abq}; shift
OUT=gpurun_out/$TAG; mkdir -p $OUT
export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests/test_gpu_multi_step.py -x -q -p no:cacheprovider --timeout 600 -k "c1_256 or shapes or partition or full_size" > $OUT/pytest.txt 2>&1; echo "pytest rc=$?" >> $OUT/pytest.txt
tail -2 $OUT/pytest.txt
bash scripts/sweep.sh $TAG "$@"
