bash tools/gpu_dev.sh "tests/test_gpu_linear.py tests/test_gpu_encoder.py tests/test_gpu_fp32.py" dbg 900
bash tools/ab.sh "ET_LIB_PATH=build/et_var_t0late/libet.so" > gpurun_out/ab.txt 2>&1
cat gpurun_out/ab.txt
