#!/bin/bash
# ncu evidence for the dominant kernel.  Usage: bash scripts/profile.sh TAG [extra bench args]
TAG=${1:-p}; shift
OUT=gpurun_out/$TAG
mkdir -p $OUT
export PYTHONUNBUFFERED=1
python -c "import __graft_entry__ as g; g.build()"
# 1) launch list of the bench command (cold-cache, serialised: compare shares, not absolutes)
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none -c 300 --csv \
  --log-file $OUT/launches.csv python bench.py --steps 2 --warmup 3 --no-extras "$@" > $OUT/launches_bench.txt 2>&1
echo "launches rc=$?"
# 2) one full capture of the top kernel (a plain and a norm iteration)
timeout 900 ncu --set full --clock-control none --import-source on -k regex:jacobi_iter -s 300 -c 2 \
  -o $OUT/prof python bench.py --steps 1 --warmup 3 --no-extras "$@" > $OUT/prof_bench.txt 2>&1
echo "full rc=$?"
ls -la $OUT
