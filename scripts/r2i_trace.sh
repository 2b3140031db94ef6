mkdir -p gpurun_out/trace7
UC_LIB_PATH=build/ab/lib_trace.so timeout 300 python scripts/trace_rounds.py > gpurun_out/trace7/trace.txt 2>&1; echo trace_rc=$?
grep -E "launch|balancing|placement|per-SM mean interior march \(us, 4" gpurun_out/trace7/trace.txt
