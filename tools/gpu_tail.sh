timeout 900 python -m pytest tests/test_gpu_encoder.py tests/test_gpu_linear.py tests/test_gpu_layernorm.py tests/test_gpu_headpar.py -q -x 2>&1 | grep -E "passed|failed|Error" | tail -5
timeout 300 python bench.py --steps 30 --warmup 5 --no-cpu-baseline --no-e2e > gpurun_out/b.json 2>gpurun_out/b.err
python -c "
import json; d=json.loads(open('gpurun_out/b.json').read().strip().splitlines()[-1]); print(round(d['value']), d['kernel_ms'], d['parity'])"
tail -3 gpurun_out/b.err
