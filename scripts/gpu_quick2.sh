#!/bin/bash
# Quick GPU check: the bench-configuration parity tests, then the default bench line.
TAG=${1:-r1q}
OUT=gpurun_out/$TAG; mkdir -p $OUT
export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests/test_gpu_jacobi.py tests/test_gpu_multi_step.py -q -p no:cacheprovider --timeout 600 \
  -k "full_size or c1_256 or switch" > $OUT/pytest.txt 2>&1; echo "pytest rc=$?" >> $OUT/pytest.txt
tail -2 $OUT/pytest.txt
timeout 600 python bench.py --steps 10 --warmup 3 > $OUT/bench.txt 2>&1; echo "bench rc=$?" >> $OUT/bench.txt
tail -2 $OUT/bench.txt | cut -c1-400
