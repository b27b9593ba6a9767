#!/bin/bash
# A/B on C4 / C5 (multi-wave grids): default build vs build/et_var_$1
mkdir -p gpurun_out
ET_LIB_PATH=build/et_var_$1/libet.so timeout 900 python -m pytest tests/test_gpu_encoder.py -x -q 2>&1 | tail -1
for v in "" "ET_LIB_PATH=build/et_var_$1/libet.so"; do
  env $v timeout 300 python bench.py --config C4 --steps 10 --warmup 3 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('C4', '${v:-default}'.ljust(40), round(d['value'],1), d['kernel_ms'], d['parity'])"
  env $v timeout 600 python bench.py --config C5 --steps 3 --warmup 2 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); print('C5', '${v:-default}'.ljust(40), round(d['value'],1), d['kernel_ms'], d['parity'])"
done
