#!/bin/bash
mkdir -p gpurun_out
timeout 900 python -m pytest tests/test_gpu_headpar.py tests/test_gpu_encoder.py -x -q 2>&1 | tail -4 > gpurun_out/hp_tests.log
timeout 600 python bench.py --parallel head --steps 10 --warmup 3 > gpurun_out/bench_hp1.json 2> gpurun_out/bench_hp1.err
mkdir -p gpurun_out/sanitizer; timeout 600 compute-sanitizer --tool racecheck --print-limit 10 python tools/sanitize_run.py C2 > gpurun_out/sanitizer/racecheck_c2_fence.log 2>&1; echo "racecheck rc $?"
cat gpurun_out/hp_tests.log; tail -c 700 gpurun_out/bench_hp1.json; tail -3 gpurun_out/bench_hp1.err; grep SUMMARY gpurun_out/sanitizer/racecheck_c2_fence.log
