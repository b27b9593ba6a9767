#!/bin/bash
# full GPU test suite, then optional sweeps (args: sweep names for tools/sweeps.py)
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -x -q 2>&1 | tail -30 > gpurun_out/gpu_tests.log
tail -5 gpurun_out/gpu_tests.log
if [ -n "$1" ]; then
  timeout 900 python tools/sweeps.py "$@" > gpurun_out/sweeps.jsonl 2> gpurun_out/sweeps.err
  cat gpurun_out/sweeps.jsonl; tail -5 gpurun_out/sweeps.err
fi
