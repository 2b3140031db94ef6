mkdir -p gpurun_out/trace8
UC_LIB_PATH=build/ab/lib_trace.so timeout 300 python scripts/trace_rounds.py --balance > gpurun_out/trace8/trace_bal.txt 2>&1; echo trace_rc=$?
head -16 gpurun_out/trace8/trace_bal.txt; grep -E "placement|per-SM mean interior march \(us, 4" gpurun_out/trace8/trace_bal.txt
