#!/bin/bash
# partial OTF: tests (watchdog + release), ncu launch times at S=1024 B=32, optional sweep
bash tools/gpu_partial.sh $1
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv python tools/partial_prof.py 1024 32 > gpurun_out/partial_ncu.csv 2>&1
grep -o '"[a-z_]*kernel<[^"]*","1","7","([0-9, ]*)","([0-9, ]*)","0","10.0","Command line profiler metrics","[a-z_.]*","[a-z]*","[0-9]*"' gpurun_out/partial_ncu.csv | tail -9 | awk -F'","' '{print $1, $9, $11}'
