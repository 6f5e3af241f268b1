bash scripts/build_variant.sh /tmp/v0.so &
bash scripts/build_variant.sh /tmp/v1.so -DDYC_FIND_MINB=4 -DDYC_UPSERT_MINB=8 -DDYC_DELETE_MINB=8 -DDYC_PLACE_MINB=8 &
bash scripts/build_variant.sh /tmp/v2.so -DDYC_FIND_MINB=3 -DDYC_UPSERT_MINB=6 -DDYC_DELETE_MINB=8 -DDYC_PLACE_MINB=6 &
wait
for v in v0 v1 v2; do for B in 4 8 16; do
  DYC_LIB=/tmp/$v.so timeout 600 python bench.py --steps 3 --warmup 2 --profile-only --bucket-slots $B > gpurun_out/bench_${v}_B$B.json 2>&1
  python -c "import json;d=json.load(open('gpurun_out/bench_${v}_B$B.json'));print('$v', $B, round(d['value']), {k:round(v) for k,v in d['ops'].items()}, d['roofline']['kernel_ms_per_step'])"
done; done
