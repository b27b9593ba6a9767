#!/bin/bash
# NEXT-2 loop: partial OTF tests under the watchdog build, then release tests + the M3/M3b sweeps
mkdir -p gpurun_out
ET_LIB_PATH=build/et_dbg/libet_dbg.so timeout 300 python -m pytest tests/test_gpu_partial.py -x -q 2>&1 | tail -30 > gpurun_out/partial_dbg.log
timeout 300 python -m pytest tests/test_gpu_partial.py tests/test_gpu_attention.py -x -q 2>&1 | tail -30 > gpurun_out/partial.log
if [ "$1" == "sweep" ]; then
  timeout 600 python tools/sweeps.py m3 m3b > gpurun_out/sweep_m3.jsonl 2> gpurun_out/sweep_m3.err
fi
tail -15 gpurun_out/partial_dbg.log; tail -15 gpurun_out/partial.log; cat gpurun_out/sweep_m3.jsonl 2>/dev/null
