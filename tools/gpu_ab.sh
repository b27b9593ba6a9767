#!/bin/bash
# A/B of variant builds: correctness of each variant on the linear/encoder tests, then tools/ab.sh.
# usage: bash tools/gpu_ab.sh NAME [NAME ...]   (build/et_var_NAME/libet.so)
mkdir -p gpurun_out
args=()
for n in "$@"; do
  ET_LIB_PATH=build/et_var_$n/libet.so timeout 600 python -m pytest tests/test_gpu_linear.py tests/test_gpu_encoder.py -x -q 2>&1 | tail -2 > gpurun_out/ab_tests_$n.log
  echo "$n: $(tail -1 gpurun_out/ab_tests_$n.log)"
  args+=("ET_LIB_PATH=build/et_var_$n/libet.so")
done
bash tools/ab.sh "${args[@]}" > gpurun_out/ab.txt 2>&1
cat gpurun_out/ab.txt
