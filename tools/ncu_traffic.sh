#!/bin/bash
# dram bytes per launch of each C3 kernel kind (ncu --set full, layer 0 of the second forward) with
# the FFN1 / FFN2 GEMMs launched separately (ET_NO_FFN_FUSE variant) so each step has its own figure.
mkdir -p gpurun_out
ET_LIB_PATH=build/et_var_nofuse/libet.so ncu --set full --clock-control none -k regex:"tsgemm|layernorm|attn" -s 84 -c 7 -f \
    -o gpurun_out/prof_traffic python tools/prof_layer.py > gpurun_out/prof_traffic.log 2>&1
python tools/ncu_summary.py gpurun_out/prof_traffic.ncu-rep > gpurun_out/ncu_traffic_v3.txt 2>&1
rm -f gpurun_out/prof_traffic.ncu-rep
cat gpurun_out/ncu_traffic_v3.txt | grep -E "^--|dram_read|dram_write|duration"
