bash scripts/build_variant.sh /tmp/u1.so -DDYC_UPSERT_U=1 -DDYC_DELETE_U=1 &
bash scripts/build_variant.sh /tmp/u4.so -DDYC_UPSERT_U=4 -DDYC_DELETE_U=4 &
timeout 1500 python -m pytest tests -m gpu -x -q -k "not full_size" 2>&1 | tail -3
wait
for v in u1 default u4; do for B in 8 16; do
  if [ $v = default ]; then L=""; else L="DYC_LIB=/tmp/$v.so"; fi
  env $L timeout 600 python bench.py --steps 3 --warmup 2 --profile-only --bucket-slots $B > gpurun_out/bench_${v}_B$B.json 2>&1
  python -c "import json;d=json.load(open('gpurun_out/bench_${v}_B$B.json'));print('$v', $B, round(d['value']), {k:round(v) for k,v in d['ops'].items()}, d['roofline']['kernel_ms_per_step'])"
done; done
