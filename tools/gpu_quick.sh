#!/bin/bash
# Quick GPU iteration: GPU tests (bounded), optional timelines, short bench.
mkdir -p gpurun_out
timeout 600 python -m pytest tests -m gpu -q -x 2>&1 | tail -15 > gpurun_out/pytest_gpu.log
if [ "$1" == "tl" ]; then
  timeout 120 python tools/gemm_timeline.py > gpurun_out/gemm_tl.txt 2>&1
  timeout 120 python tools/attn_timeline.py > gpurun_out/attn_tl.txt 2>&1
fi
timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
cat gpurun_out/pytest_gpu.log
python - <<'PY'
import json
try:
    d = json.loads(open("gpurun_out/bench.json").read().strip().splitlines()[-1])
    print("value", round(d["value"]), "ms", round(d["ms_per_step"], 4), "kernel_ms", d["kernel_ms"], "clocks", d["clocks"]["sm_mhz"], d["clocks"]["reasons"])
except Exception as e:
    print("bench failed", e); print(open("gpurun_out/bench.err").read()[-3000:])
PY
