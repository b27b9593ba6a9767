ncu --set full --cache-control none --clock-control none -k regex:layernorm -s 20 -c 2 -f -o gpurun_out/prof_ln_warm python tools/ln_probe.py > gpurun_out/prof_ln_warm.log 2>&1
python tools/ncu_summary.py gpurun_out/prof_ln_warm.ncu-rep > gpurun_out/ncu_ln_warm.txt 2>&1
ncu -i gpurun_out/prof_ln_warm.ncu-rep --page details --csv 2>/dev/null | grep -i -E "Memory Throughput|DRAM Through|L2 Hit|L1/TEX Hit|Duration|Achieved Occupancy|Mem Busy|Max Bandwidth|L2 Cache Throughput|Registers|Waves Per SM|Block Limit" > gpurun_out/ncu_ln_warm_details.txt
rm -f gpurun_out/prof_ln_warm.ncu-rep
