#!/bin/bash
# A/B of grouped skew (UC_SKEW=S: groups of S levels): variant-5 parity, then the sweep.
OUT=gpurun_out/skew3; mkdir -p $OUT
export PYTHONUNBUFFERED=1
for lib in skew3 skew2; do
  UC_LIB_PATH=build/ab/$lib.so timeout 900 python -m pytest tests/test_gpu_multi_step.py -x -q -p no:cacheprovider --timeout 600 \
    -k "c1_256 or shapes or partition or full_size" > $OUT/pytest_$lib.txt 2>&1; echo "pytest $lib rc=$?" >> $OUT/pytest_$lib.txt
  tail -2 $OUT/pytest_$lib.txt
done
bash scripts/sweep.sh skew3 "-|" "skew3|" "skew2|" "-|" "skew3|" "skew2|" "skew3|--tile-rows 8" "skew2|--tile-rows 8" "skew3|--tile-rows 7" "skew2|--tile-rows 5"
