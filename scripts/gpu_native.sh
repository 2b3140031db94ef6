#!/bin/bash
# NCCL device-API comparator: parity vs the oracle, then its timing at the bench workload.
OUT=gpurun_out/native; mkdir -p $OUT
export PYTHONUNBUFFERED=1
timeout 600 python -m pytest tests/test_gpu_native.py -q -p no:cacheprovider --timeout 300 > $OUT/pytest.txt 2>&1; echo "pytest rc=$?" >> $OUT/pytest.txt
tail -15 $OUT/pytest.txt
NCCL_DEBUG=WARN timeout 300 python benchmarks/nccl_dev_bench.py > $OUT/bench.txt 2>&1; echo "bench rc=$?" >> $OUT/bench.txt
tail -3 $OUT/bench.txt
timeout 300 python benchmarks/nccl_dev_bench.py --nx 4096 --ny 4096 --iters 1000 >> $OUT/bench.txt 2>&1
tail -1 $OUT/bench.txt
