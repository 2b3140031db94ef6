#!/bin/bash
# ncu evidence for the CG workload.  Usage: bash scripts/profile_cg.sh TAG
TAG=${1:-pcg}; OUT=gpurun_out/$TAG; mkdir -p $OUT
timeout 900 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none \
  -k regex:cg_ -s 30 -c 30 --csv --log-file $OUT/launches.csv \
  python benchmarks/cg_bench.py --grid 160 --iters 10 --steps 1 --warmup 1 --cpu-iters 0 > $OUT/launches_bench.txt 2>&1
echo "launches rc=$?"
timeout 900 ncu --set full --clock-control none --import-source on -k regex:cg_spmv -s 10 -c 1 -o $OUT/prof \
  python benchmarks/cg_bench.py --grid 160 --iters 10 --steps 1 --warmup 1 --cpu-iters 0 > $OUT/prof_bench.txt 2>&1
echo "full rc=$?"
