timeout 1500 python -m pytest tests -m gpu -x -q -k "not full_size" 2>&1 | tail -3
bash scripts/gpu_streams2.sh
timeout 600 python bench.py --steps 5 --warmup 3 --profile-only > gpurun_out/b18.json 2> gpurun_out/b18.err; tail -3 gpurun_out/b18.err
python -c "import json;d=json.load(open('gpurun_out/b18.json'));print(round(d['value']), d['ms_per_step'], {k:round(v) for k,v in d['ops'].items()}, d['roofline']['kernel_ms_per_step'])"
