timeout 1500 python -m pytest tests -m gpu -x -q -k "not full_size" 2>&1 | tail -5
for B in 4 8 16; do
  timeout 600 python bench.py --steps 3 --warmup 2 --profile-only --bucket-slots $B > gpurun_out/bench_B$B.json 2>&1
  python -c "import json;d=json.load(open('gpurun_out/bench_B$B.json'));print($B, round(d['value']), {k:round(v) for k,v in d['ops'].items()}, d['roofline']['kernel_ms_per_step'], d['table'])"
done
