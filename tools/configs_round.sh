#!/bin/bash
# every BASELINE config on one GPU (bench lines into gpurun_out/bench_<C>.json)
mkdir -p gpurun_out
for c in C1 C2 C3 C4; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
timeout 900 python bench.py --config C5 --steps 5 --warmup 3 > gpurun_out/bench_C5.json 2> gpurun_out/bench_C5.err
for c in C1 C2 C3 C4 C5; do python - <<PY
import json
try:
    d=json.loads(open("gpurun_out/bench_$c.json").read().strip().splitlines()[-1])
    print("$c", round(d["value"],1), d["unit"], "ms", round(d["ms_per_step"],4), "roof", d["roofline"]["kernel"], round(d["roofline"]["frac"],3), "ns", round(d["north_star"]["frac_of_measured_tc_burst"],3), "stepwise", round(d["stepwise_roofline_frac"],3), "parity", d.get("parity",{}).get("max_abs"), "e2e", round(d["e2e"]["value"],1), d["scaling"])
except Exception as e:
    print("$c failed", e, open("gpurun_out/bench_$c.err").read()[-1500:])
PY
done
