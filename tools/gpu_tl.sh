#!/bin/bash
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q -rA -s -k "full_depth" 2>&1 | grep -E "full depth|passed|failed|Error" | tail -8 > gpurun_out/fulldepth.log
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -8 > gpurun_out/dev.log
timeout 300 python bench.py --steps 20 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/bench.json 2> gpurun_out/bench.err
python -c "
import json
d=json.loads(open('gpurun_out/bench.json').read().strip().splitlines()[-1]); print(round(d['value']), d['kernel_ms'], d['parity'])"
cat gpurun_out/fulldepth.log gpurun_out/dev.log
