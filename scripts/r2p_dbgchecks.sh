# the GPU suite against the bounds-checked build (UC_DEBUG_CHECKS: device asserts on rows read, ring
# offsets, balanced tables; compute-sanitizer is closed on this pool)
set -x
O=gpurun_out/dbg; mkdir -p $O
UC_LIB_PATH=build/ab/lib_dbg.so timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -x > $O/pytest_dbg.log 2>&1; echo pytest_dbg_rc=$?
tail -5 $O/pytest_dbg.log
grep -c "UC_CHECK failed" $O/pytest_dbg.log
