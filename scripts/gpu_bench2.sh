#!/bin/bash
export PYTHONUNBUFFERED=1
mkdir -p gpurun_out/b2
timeout 600 python bench.py --steps 10 --warmup 3 > gpurun_out/b2/bench.txt 2>&1; tail -1 gpurun_out/b2/bench.txt
timeout 600 python bench.py --steps 10 --warmup 3 --ny-per-gpu 2048 > gpurun_out/b2/bench_2048.txt 2>&1; tail -1 gpurun_out/b2/bench_2048.txt
timeout 600 python bench.py --steps 10 --warmup 3 --variant 1 --ny-per-gpu 2048 --no-extras > gpurun_out/b2/bench_2048_v1.txt 2>&1; tail -1 gpurun_out/b2/bench_2048_v1.txt
timeout 600 python bench.py --steps 10 --warmup 3 --mode host --no-extras > gpurun_out/b2/bench_host.txt 2>&1; tail -1 gpurun_out/b2/bench_host.txt
timeout 600 python bench.py --steps 10 --warmup 3 --mode host --variant 1 --no-extras > gpurun_out/b2/bench_host_v1.txt 2>&1; tail -1 gpurun_out/b2/bench_host_v1.txt
timeout 900 python -m pytest tests/test_gpu_multi_step.py tests/test_gpu_fullsize.py -q -x --timeout 600 -p no:cacheprovider > gpurun_out/b2/pytest.txt 2>&1; tail -2 gpurun_out/b2/pytest.txt
