#!/bin/bash
# Two-ghost-lane layout (T = 5..8 iterations per launch): parity, then the A/B sweep at the bench workload.
OUT=gpurun_out/t8; mkdir -p $OUT
export PYTHONUNBUFFERED=1
timeout 1200 python -m pytest tests/test_gpu_multi_step.py -x -q -p no:cacheprovider --timeout 600 > $OUT/pytest.txt 2>&1; echo "pytest rc=$?" >> $OUT/pytest.txt
tail -3 $OUT/pytest.txt
bash scripts/sweep.sh t8 "-|" "-|--tile-rows 8" "-|--tile-rows 8 --block-x 256" "-|--tile-rows 8 --stages 12" \
  "-|--tile-rows 8 --block-x 256 --stages 12" "-|--tile-rows 6" "-|--tile-rows 5" "-|--tile-rows 7" "-|--tile-rows 8 --stages 16" \
  "-|--tile-rows 8 --block-x 192 --stages 12"
