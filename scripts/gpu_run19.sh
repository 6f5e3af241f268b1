timeout 1500 python -m pytest tests -m gpu -x -q -k "not full_size" 2>&1 | tail -3
bash scripts/gpu_c5b.sh
timeout 600 python bench.py --steps 5 --warmup 3 --no-cpu-baseline --no-e2e > gpurun_out/b19.json 2> gpurun_out/b19.err; tail -3 gpurun_out/b19.err
python -c "import json;d=json.load(open('gpurun_out/b19.json'));print(round(d['value']), d['ms_per_step'], {k:round(v) for k,v in d['ops'].items()}, d['roofline']['kernel_ms_per_step'], d['resize'])"
