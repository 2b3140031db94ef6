# A/B of the march builds on the full product kernel (bench --no-extras) + ncu of the product <6,2>
set -x
T=${1:-ab}
mkdir -p gpurun_out/$T
for i in 1 2; do
  timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_product_$i.log 2>&1
  UC_LIB_PATH=build/ab/lib_nogroup.so timeout 300 python bench.py --no-extras --steps 10 --stages 8 > gpurun_out/$T/bench_nogroup_$i.log 2>&1
  UC_LIB_PATH=build/ab/lib_g9_nota.so timeout 300 python bench.py --no-extras --steps 10 > gpurun_out/$T/bench_g9nota_$i.log 2>&1
done
for f in gpurun_out/$T/bench_*.log; do echo "$f $(tail -1 $f | python -c 'import json,sys; d=json.loads(sys.stdin.read()); print(d["value"], d["roofline"]["kernel_ms"])' 2>&1)"; done
LIST=scripts/proto/list_ta.txt bash scripts/proto/run_bm2.sh ta
timeout 600 ncu --set full --clock-control none --import-source on -k regex:jacobi_t_kernel -s 5 -c 1 -o gpurun_out/$T/t6_product python bench.py --steps 1 --warmup 3 --no-extras > gpurun_out/$T/ncu.log 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q -p no:cacheprovider -k "host_paths or solve or lifecycle or put_signal_ring or concurrent" > gpurun_out/$T/pytest.log 2>&1; echo pytest_rc=$?
tail -3 gpurun_out/$T/pytest.log
