#!/bin/bash
# One ncu --set full capture of a kernel.  Usage: bash scripts/profile_kernel.sh TAG REGEX SKIP [bench args]
TAG=${1:-p}; RX=${2:-jacobi}; SKIP=${3:-100}; shift 3
OUT=gpurun_out/$TAG
mkdir -p $OUT
export PYTHONUNBUFFERED=1
python -c "import __graft_entry__ as g; g.build()" > $OUT/build.txt 2>&1
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$RX -s $SKIP -c 2 \
  -o $OUT/prof python bench.py --steps 1 --warmup 3 --no-extras "$@" > $OUT/prof_bench.txt 2>&1
echo "full rc=$?"
ls -la $OUT
