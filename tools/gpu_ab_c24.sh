#!/bin/bash
# A/B on C2 and C4 (attention-aware configs): default build vs build/et_var_$1
mkdir -p gpurun_out
ET_LIB_PATH=build/et_var_$1/libet.so timeout 600 python -m pytest tests/test_gpu_encoder.py tests/test_gpu_attention.py -x -q 2>&1 | tail -1
for i in 1 2; do for v in "" "ET_LIB_PATH=build/et_var_$1/libet.so"; do for c in C2 C4; do
  env $v timeout 300 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline --no-e2e --no-parity 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('$c', '${v:-default}'.ljust(40), round(d['value']), round(d['kernel_ms']['attention']*1e3,2))"
done; done; done
