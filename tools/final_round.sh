#!/bin/bash
# Round-end evidence on one GPU: full GPU test suite, the default bench line (C3), the reference arm,
# the other configs' lines, the ncu launch list + full-set summaries, and the GEMM cycle timeline.
mkdir -p gpurun_out
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -15 > gpurun_out/gpu_tests.log
timeout 900 python bench.py > gpurun_out/bench_c3_final.json 2> gpurun_out/bench_c3_final.err
timeout 600 python bench.py --impl reference --steps 3 --warmup 1 > gpurun_out/bench_c3_reference.json 2> gpurun_out/bench_ref.err
for c in C1 C2 C4; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
timeout 900 python bench.py --config C5 --steps 5 --warmup 3 > gpurun_out/bench_C5.json 2> gpurun_out/bench_C5.err
bash tools/profile_round.sh > /dev/null 2>&1
ET_LIB_PATH=build/et_dbg/libet_dbg.so timeout 300 python tools/gemm_timeline.py > gpurun_out/gemm_tl.txt 2>&1
tail -3 gpurun_out/gpu_tests.log
for f in gpurun_out/bench_c3_final.json gpurun_out/bench_C1.json gpurun_out/bench_C2.json gpurun_out/bench_C4.json gpurun_out/bench_C5.json gpurun_out/bench_c3_reference.json; do
  python - "$f" <<'PY'
import json, sys
f = sys.argv[1]
try:
    d = json.loads(open(f).read().strip().splitlines()[-1])
    print(f, round(d["value"], 2), d["unit"], d.get("ms_per_step"), d.get("roofline", {}).get("kernel"), d.get("roofline", {}).get("frac"), d.get("parity", {}).get("max_abs"))
except Exception as e:
    print(f, "failed", e)
PY
done
