#!/bin/bash
# Last check of the committed state on one GPU: full GPU suite, smoke(), the default bench line.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -3 > gpurun_out/gpu_tests_final.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/smoke_final.log 2>&1
timeout 900 python bench.py > gpurun_out/bench_c3_final.json 2> gpurun_out/bench_c3_final.err
timeout 600 python bench.py --config C2 --steps 20 --warmup 3 > gpurun_out/bench_c2_final.json 2> gpurun_out/bench_c2_final.err
timeout 600 python bench.py --config C4 --steps 20 --warmup 3 > gpurun_out/bench_c4_final.json 2> gpurun_out/bench_c4_final.err
cat gpurun_out/gpu_tests_final.log; tail -1 gpurun_out/smoke_final.log
for f in gpurun_out/bench_c3_final.json gpurun_out/bench_c2_final.json gpurun_out/bench_c4_final.json; do
python - "$f" <<'PY'
import json, sys
d = json.loads(open(sys.argv[1]).read().strip().splitlines()[-1])
print(sys.argv[1], round(d["value"], 1), d["ms_per_step"], d["e2e"]["value"], d["roofline"]["frac"], d["parity"]["max_abs"], d["clocks"]["sm_mhz"], d["clocks"]["reasons"])
PY
done
