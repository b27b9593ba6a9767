#!/bin/bash
# development loop: selected GPU tests (debug build with mbarrier watchdog first if asked), then bench
mkdir -p gpurun_out
SEL=${1:-"tests/test_gpu_linear.py"}
if [ "$2" == "dbg" ]; then
  ET_LIB_PATH=build/et_dbg/libet_dbg.so timeout 240 python -m pytest $SEL -x -q 2>&1 | tail -40 > gpurun_out/dev_dbg.log
fi
timeout ${3:-600} python -m pytest $SEL -x -q 2>&1 | tail -40 > gpurun_out/dev.log
if [ "$4" == "bench" ]; then
  timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
fi
cat gpurun_out/dev_dbg.log 2>/dev/null | tail -15; cat gpurun_out/dev.log | tail -25
