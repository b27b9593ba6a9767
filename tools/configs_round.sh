#!/bin/bash
# Bench lines for the other BASELINE configs (parity configs, not the headline): C2, C4, C5 (1 GPU).
mkdir -p gpurun_out
for c in C2 C4; do
  timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline > gpurun_out/bench_$c.json 2> gpurun_out/bench_$c.err
done
timeout 900 python bench.py --config C5 --steps 3 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/bench_C5.json 2> gpurun_out/bench_C5.err
timeout 600 python bench.py --parallel head --steps 20 --warmup 3 > gpurun_out/bench_hp1.json 2> gpurun_out/bench_hp1.err
tail -c 600 gpurun_out/bench_*.err
