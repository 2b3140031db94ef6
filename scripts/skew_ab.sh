#!/bin/bash
# A/B of the skewed level schedule (UC_SKEW=1): variant-5 parity on the skew builds, then the sweep.
OUT=gpurun_out/skew; mkdir -p $OUT
export PYTHONUNBUFFERED=1
for lib in skew_256m1 skew_384m1; do
  UC_LIB_PATH=build/ab/$lib.so timeout 900 python -m pytest tests/test_gpu_multi_step.py -x -q -p no:cacheprovider --timeout 600 \
    -k "c1_256 or shapes or partition or full_size" > $OUT/pytest_$lib.txt 2>&1; echo "pytest $lib rc=$?" >> $OUT/pytest_$lib.txt
  tail -2 $OUT/pytest_$lib.txt
done
bash scripts/sweep.sh skew "-|" "skew_256m1|" "skew_384m1|" "-|" "skew_256m1|" "skew_384m1|" "skew_256m1|--tile-rows 8" "skew_384m1|--tile-rows 8" "skew_256m1|--tile-rows 7" "skew_384m1|--tile-rows 7"
