#!/bin/bash
# usage (on the GPU box): bash scripts/probe/run.sh
set -x
mkdir -p gpurun_out
nvidia-smi > gpurun_out/probe_nvsmi.txt 2>&1
nvidia-smi topo -m >> gpurun_out/probe_nvsmi.txt 2>&1
lscpu | head -20 > gpurun_out/probe_lscpu.txt; nproc >> gpurun_out/probe_lscpu.txt
timeout 60 ./scripts/probe/probe > gpurun_out/probe.txt 2>&1; echo "rc=$?" >> gpurun_out/probe.txt; timeout 30 ./scripts/probe/probe ipc > gpurun_out/probe_ipc.txt 2>&1; echo "rc=$?" >> gpurun_out/probe_ipc.txt
cat gpurun_out/probe.txt
