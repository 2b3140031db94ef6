#!/bin/bash
# quick check: variant-5 parity + two bench lines.  Usage: bash scripts/gpu_quick.sh TAG [pytest -k expr]
TAG=${1:-q}; OUT=gpurun_out/$TAG; mkdir -p $OUT
export PYTHONUNBUFFERED=1
timeout 900 python -m pytest tests/test_gpu_multi_step.py -q -x --timeout 300 -p no:cacheprovider > $OUT/pytest.txt 2>&1; tail -2 $OUT/pytest.txt
for i in 1 2; do timeout 300 python bench.py --steps 20 --warmup 3 --no-extras 2>&1 | tail -1 | python -c "
import json,sys; d=json.loads(sys.stdin.read()); r=d['roofline']; print('GLUPS', d['value'], 'kernel_ms', r['kernel_ms'], 'frac', r['frac'], 'norm_ms', r['kernel_norm_ms'], d['clocks'])"; done
