# Binned path: parity tests, then the C2 bench (auto = binned) and the direct kernels for comparison.
timeout 900 python -m pytest tests/test_gpu_binned.py -x -q 2>&1 | tail -15
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e --no-rehash > gpurun_out/bin1_bench.json 2> gpurun_out/bin1_bench.err; tail -3 gpurun_out/bin1_bench.err
python - <<'PY'
import json
d=json.load(open('gpurun_out/bin1_bench.json'))
print(d['value'], d['ms_per_step'], d['phase_ms'], d['ops'])
print(d['roofline'].get('kernel_ms_per_step'))
PY
