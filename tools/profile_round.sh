#!/bin/bash
# Run on the GPU box (gpurun): the default bench line, the ncu launch list of a short bench run, and
# one `ncu --set full` capture per kernel kind of the C3 encoder's second call, summarised on the box
# (tools/ncu_summary.py); the LayerNorm report is summarised and dropped (tens of MB).  Output: gpurun_out/.
mkdir -p gpurun_out
timeout 900 python bench.py > gpurun_out/bench_full.json 2> gpurun_out/bench_full.err
ncu --metrics gpu__time_duration.sum --clock-control none -c 2500 --csv --log-file gpurun_out/launches.csv \
    python bench.py --steps 2 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/launches_bench.log 2>&1
# 84 kernel launches per encoder call (12 layers x 7); the second call's layer-0 kernels
ncu --set full --clock-control none --import-source on -k regex:tsgemm -s 48 -c 4 -f -o gpurun_out/prof_gemm \
    python tools/prof_layer.py > gpurun_out/prof_gemm.log 2>&1
ncu --set full --clock-control none --import-source on -k regex:attn -s 12 -c 1 -f -o gpurun_out/prof_attn \
    python tools/prof_layer.py > gpurun_out/prof_attn.log 2>&1
ncu --set full --clock-control none -k regex:layernorm -s 24 -c 2 -f -o gpurun_out/prof_ln \
    python tools/prof_layer.py > gpurun_out/prof_ln.log 2>&1
python tools/ncu_summary.py gpurun_out/prof_gemm.ncu-rep gpurun_out/prof_attn.ncu-rep gpurun_out/prof_ln.ncu-rep \
    > gpurun_out/ncu_summary.txt 2>&1
rm -f gpurun_out/prof_ln.ncu-rep
ls -la gpurun_out
