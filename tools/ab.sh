#!/bin/bash
# A/B bench: the default build vs env-var variants, 3 alternating runs each (short bench lines).
mkdir -p gpurun_out
for i in 1 2 3; do
  for v in "" "$@"; do
    env $v timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e 2>/dev/null | python -c "
import json,sys
d=json.loads(sys.stdin.read().strip().splitlines()[-1]); k=d['kernel_ms']
print('${v:-default}'.ljust(24), round(d['value']), ' '.join(f'{n}={v*1e3:.2f}' for n,v in k.items()))"
  done
done
