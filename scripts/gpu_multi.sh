#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out/ms1
timeout 1200 python -m pytest tests/test_gpu_multi_step.py -x -q --timeout 300 -p no:cacheprovider > gpurun_out/ms1/pytest.txt 2>&1; echo "rc=$?" >> gpurun_out/ms1/pytest.txt
tail -40 gpurun_out/ms1/pytest.txt
for T in 1 2 3 4; do timeout 300 python bench.py --steps 5 --warmup 3 --variant 5 --tile-rows $T --no-extras 2>&1 | tail -1 | cut -c1-400; done
