#!/bin/bash
# ncu --set full of one kernel from an A/B build.  Usage: bash scripts/profile_ab.sh TAG LIB REGEX SKIP [bench args]
TAG=$1; LIB=$2; RX=$3; SKIP=$4; shift 4
OUT=gpurun_out/$TAG; mkdir -p $OUT
export PYTHONUNBUFFERED=1
[ "$LIB" != "-" ] && export UC_LIB_PATH=build/ab/$LIB.so
timeout 900 ncu --set full --clock-control none --import-source on -k regex:$RX -s $SKIP -c 2 \
  -o $OUT/prof python bench.py --steps 1 --warmup 3 --no-extras "$@" > $OUT/prof_bench.txt 2>&1
echo "full rc=$?"; ls -la $OUT
