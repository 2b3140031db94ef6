#!/bin/bash
# ncu --set full of one variant-5 launch.  Usage: profile_t6.sh TAG LIB(- = product) bench-args...
TAG=$1; LIB=$2; shift 2
OUT=gpurun_out/$TAG; mkdir -p $OUT
if [ "$LIB" != "-" ]; then export UC_LIB_PATH=build/ab/$LIB.so; fi
timeout 900 ncu --set full --clock-control none --import-source on -k regex:jacobi_t_kernel -s 40 -c 1 \
  -o $OUT/prof python bench.py --steps 1 --warmup 3 --no-extras "$@" > $OUT/prof.txt 2>&1; echo "rc=$?"
ls -la $OUT
