#!/bin/bash
# Full GPU session: tests, smoke, ncu launch list + full capture of the dominant kernel, bench.
TAG=${1:-r1d}
OUT=gpurun_out/$TAG
mkdir -p $OUT
export PYTHONUNBUFFERED=1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1; echo "build rc=$?" >> $OUT/build.txt
timeout 1800 python -m pytest tests -m gpu -q --timeout 600 -p no:cacheprovider > $OUT/pytest_gpu.txt 2>&1; echo "pytest rc=$?" >> $OUT/pytest_gpu.txt
tail -5 $OUT/pytest_gpu.txt
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $OUT/smoke.txt 2>&1; echo "smoke rc=$?" >> $OUT/smoke.txt
tail -2 $OUT/smoke.txt
timeout 600 python bench.py --steps 10 --warmup 3 > $OUT/bench.txt 2>&1; echo "bench rc=$?" >> $OUT/bench.txt
tail -3 $OUT/bench.txt
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 400 --csv \
  --log-file $OUT/launches.csv python bench.py --steps 2 --warmup 3 --no-extras > $OUT/launches_bench.txt 2>&1
echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:jacobi_t_kernel -s 80 -c 1 \
  -o $OUT/prof python bench.py --steps 1 --warmup 3 --no-extras > $OUT/prof_bench.txt 2>&1
echo "full rc=$?"
