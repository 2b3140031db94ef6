export PYTHONUNBUFFERED=1
mkdir -p gpurun_out/ts1
timeout 900 python -m pytest tests/test_gpu_two_step.py -x -q --timeout 300 -p no:cacheprovider > gpurun_out/ts1/pytest_two_step.txt 2>&1; echo "rc=$?" >> gpurun_out/ts1/pytest_two_step.txt
tail -30 gpurun_out/ts1/pytest_two_step.txt
timeout 300 python bench.py --steps 10 --warmup 3 --variant 4 --no-extras > gpurun_out/ts1/bench_v4.txt 2>&1; tail -2 gpurun_out/ts1/bench_v4.txt
timeout 300 python bench.py --steps 10 --warmup 3 --no-extras > gpurun_out/ts1/bench_v1.txt 2>&1; tail -2 gpurun_out/ts1/bench_v1.txt
