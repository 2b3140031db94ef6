# A/B of the PQ register frame (product) vs the natural frame (UC_PQ_FRAME=0) vs PQ with move
# permutation (UC_PQ_ADD_PERMUTE=0); parity subset on the product build; FP32 pipe-rate probe
set -x
T=${1:-pq}
mkdir -p gpurun_out/$T
(cd scripts/probe && nvcc -gencode arch=compute_100a,code=sm_100a -O3 -o pipes pipes.cu && ./pipes) > gpurun_out/$T/pipes.txt 2>&1
python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/$T/smoke.log 2>&1; echo smoke_rc=$?
for i in 1 2; do
  timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_pq_$i.log 2>&1
  UC_LIB_PATH=build/ab/lib_pq0.so timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_nat_$i.log 2>&1
  UC_LIB_PATH=build/ab/lib_pqmov.so timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_pqmov_$i.log 2>&1
done
for st in 18 27; do timeout 300 python bench.py --no-extras --steps 10 --stages $st > gpurun_out/$T/bench_pq_st$st.log 2>&1; done
for f in gpurun_out/$T/bench_*.log; do echo "$f $(tail -1 $f | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"], d["clocks"]["sm_mhz"])' 2>&1)"; done
timeout 1500 python -m pytest tests/test_gpu_multi_step.py tests/test_gpu_jacobi.py -x -q -p no:cacheprovider > gpurun_out/$T/pytest.log 2>&1; echo pytest_rc=$?
tail -3 gpurun_out/$T/pytest.log
