# NEXT-4 (d sensitivity) and static fill sweep (Fig. fig:static-filled-factor)
for d in 2 3 4 5 6 8; do
  timeout 600 python bench.py --d $d --steps 3 --warmup 2 --profile-only > gpurun_out/sw_d$d.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/sw_d$d.json'));print('d=$d', round(d['value']), {k:round(v) for k,v in d['ops'].items()}, round(d['roofline']['model']['phi'],3), round(d['roofline']['model']['evictions_per_insert'],3))"
done
for th in 0.70 0.75 0.80 0.85 0.90; do
  timeout 600 python bench.py --beta $th --steps 3 --warmup 2 --profile-only > gpurun_out/sw_t$th.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/sw_t$th.json'));print('theta=$th', round(d['value']), {k:round(v) for k,v in d['ops'].items()}, round(d['table']['fill_after_insert'],3), round(d['roofline']['model']['phi'],3))"
done
# NEXT-2 dynamic sweeps on C3 (TW shape, scale 0.25): r, alpha, beta, batch
for r in 0.1 0.3 0.5; do
  timeout 900 python bench.py --config c3 --scale 0.25 --r $r --warmup 1 > gpurun_out/sw_c3_r$r.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/sw_c3_r$r.json'));print('c3 r=$r', round(d['value']), {k:round(v) for k,v in d['ops'].items()}, d['fill_track']['min_after_mutation'], d['fill_track']['max'], d['table_bytes']['max'])"
done
for a in 0.2 0.4; do
  timeout 900 python bench.py --config c3 --scale 0.25 --alpha $a --warmup 1 > gpurun_out/sw_c3_a$a.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/sw_c3_a$a.json'));print('c3 alpha=$a', round(d['value']), {k:round(v) for k,v in d['ops'].items()}, d['fill_track']['min_after_mutation'], d['fill_track']['max'], d['table_bytes']['max'])"
done
for b in 0.7 0.9; do
  timeout 900 python bench.py --config c3 --scale 0.25 --beta $b --warmup 1 > gpurun_out/sw_c3_b$b.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/sw_c3_b$b.json'));print('c3 beta=$b', round(d['value']), {k:round(v) for k,v in d['ops'].items()}, d['fill_track']['min_after_mutation'], d['fill_track']['max'], d['table_bytes']['max'])"
done
for bs in 200000 600000; do
  timeout 900 python bench.py --config c3 --scale 0.25 --batch $bs --warmup 1 > gpurun_out/sw_c3_bs$bs.json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/sw_c3_bs$bs.json'));print('c3 batch=$bs', round(d['value']), {k:round(v) for k,v in d['ops'].items()}, d['fill_track']['min_after_mutation'], d['fill_track']['max'])"
done
