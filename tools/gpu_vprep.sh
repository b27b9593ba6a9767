timeout 900 python -m pytest tests/test_gpu_encoder.py tests/test_gpu_headpar.py tests/test_gpu_attention.py tests/test_gpu_precomputed.py -q 2>&1 | grep -E "passed|failed|Error" | tail -6
for c in C2 C4; do timeout 600 python bench.py --config $c --steps 20 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b_$c.json 2> gpurun_out/b_$c.err; python -c "
import json; d=json.loads(open('gpurun_out/b_$c.json').read().strip().splitlines()[-1]); print('$c', round(d['value'],1), d['ms_per_step'], d['gpu_launches']/d['steps'], d['kernel_ms'], d['parity'])"; done
