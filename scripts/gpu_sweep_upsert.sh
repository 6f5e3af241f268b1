i=0
for cfg in "2 1" "2 4" "4 1" "4 3" "4 4" "8 2"; do
  set -- $cfg
  bash scripts/build_variant.sh /tmp/s_$1_$2.so -DDYC_UPSERT_U=$1 -DDYC_UPSERT_MINB=$2 &
done
wait
for cfg in "2 1" "2 4" "4 1" "4 3" "4 4" "8 2"; do
  set -- $cfg
  DYC_LIB=/tmp/s_$1_$2.so timeout 600 python bench.py --steps 3 --warmup 2 --profile-only > gpurun_out/sw_$1_$2.json 2>&1
  python -c "import json;d=json.load(open('gpurun_out/sw_$1_$2.json'));print('U=$1 minb=$2', round(d['value']), {k:round(v) for k,v in d['ops'].items()}, d['roofline']['kernel_ms_per_step'])"
done
