for cfg in "2 4" "4 4" "2 2" "2 8" "4 8"; do
  set -- $cfg
  bash scripts/build_variant.sh /tmp/d_$1_$2.so -DDYC_DELETE_U=$1 -DDYC_FIND_ILP=$2 &
done
wait
for cfg in "2 4" "4 4" "2 2" "2 8" "4 8"; do
  set -- $cfg
  DYC_LIB=/tmp/d_$1_$2.so timeout 600 python bench.py --steps 3 --warmup 2 --profile-only > gpurun_out/sw2_$1_$2.json 2>&1
  python -c "import json;d=json.load(open('gpurun_out/sw2_$1_$2.json'));print('delU=$1 findILP=$2', round(d['value']), {k:round(v) for k,v in d['ops'].items()}, d['roofline']['kernel_ms_per_step'])"
done
