#!/bin/bash
OUT=gpurun_out/repro; mkdir -p $OUT
for i in 1 2 3; do
  timeout 300 python -m pytest tests/test_gpu_jacobi.py -q -p no:cacheprovider -k "graph_and_stepwise" 2>&1 | tail -1 | sed "s/^/product $i: /" | tee -a $OUT/log.txt
  UC_LIB_PATH=build/ab/nohoist.so timeout 300 python -m pytest tests/test_gpu_jacobi.py -q -p no:cacheprovider -k "graph_and_stepwise" 2>&1 | tail -1 | sed "s/^/nohoist $i: /" | tee -a $OUT/log.txt
done
