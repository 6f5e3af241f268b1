timeout 600 python bench.py --d 2 --steps 3 --warmup 2 --profile-only > gpurun_out/sw_d2.json 2> gpurun_out/sw_d2.err; tail -5 gpurun_out/sw_d2.err
python -c "import json;d=json.load(open('gpurun_out/sw_d2.json'));print('d=2', round(d['value']), {k:round(v) for k,v in d['ops'].items()}, round(d['roofline']['model']['phi'],3), round(d['roofline']['model']['evictions_per_insert'],3))"
for th in 0.70 0.75 0.80 0.85 0.90; do
  timeout 600 python bench.py --beta $th --alpha 0.1 --steps 3 --warmup 2 --profile-only > gpurun_out/sw_t$th.json 2> gpurun_out/sw_t.err; tail -2 gpurun_out/sw_t.err
  python -c "import json;d=json.load(open('gpurun_out/sw_t$th.json'));print('theta=$th', round(d['value']), {k:round(v) for k,v in d['ops'].items()}, round(d['table']['fill_after_insert'],3), round(d['roofline']['model']['phi'],3), round(d['roofline']['model']['evictions_per_insert'],3))"
done
