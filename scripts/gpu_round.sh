#!/bin/bash
# One GPU session: tests, smoke, bench, ncu.  Usage: bash scripts/gpu_round.sh [tag]
TAG=${1:-r1}
OUT=gpurun_out/$TAG
mkdir -p $OUT
export PYTHONUNBUFFERED=1
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,power.draw --format=csv > $OUT/nvsmi.txt 2>&1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1; echo "build rc=$?" >> $OUT/build.txt
timeout 1500 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.txt
tail -5 $OUT/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1; echo "smoke rc=$?" >> $OUT/smoke.txt
tail -2 $OUT/smoke.txt
timeout 600 python bench.py --steps 10 --warmup 3 > $OUT/bench.txt 2>&1; echo "bench rc=$?" >> $OUT/bench.txt
tail -3 $OUT/bench.txt
