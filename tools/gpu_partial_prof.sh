bash tools/gpu_partial.sh
ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none --csv python tools/partial_prof.py 1024 32 > gpurun_out/partial_ncu.csv 2>&1
tail -8 gpurun_out/partial_ncu.csv
