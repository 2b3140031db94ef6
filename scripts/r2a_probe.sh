set -x
mkdir -p gpurun_out/r2a
nvidia-smi -L
python -c "import paper_conf_cluster_sagbilieinu25_b200 as U; print(U.lib.uc_version())"
timeout 600 ncu --set full --clock-control none --import-source on -k regex:jacobi_t_kernel -s 5 -c 1 -o gpurun_out/r2a/t6 python bench.py --steps 1 --warmup 3 --no-extras > gpurun_out/r2a/ncu.log 2>&1
echo ncu_rc=$?
timeout 300 python bench.py --steps 10 --warmup 3 --no-extras > gpurun_out/r2a/bench.log 2>&1
echo bench_rc=$?
for t in memcheck synccheck racecheck; do UC_SANITIZE_T6_ONLY=1 timeout 900 compute-sanitizer --tool $t python scripts/sanitize_run.py > gpurun_out/r2a/san_$t.log 2>&1; echo "$t rc=$?" >> gpurun_out/r2a/san_rc.txt; done
cat gpurun_out/r2a/san_rc.txt
tail -3 gpurun_out/r2a/bench.log
