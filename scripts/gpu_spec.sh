for v in spec0_u4 spec1_u2 spec1_u3 spec1_u4; do
  DYC_LIB=variants/v_$v.so timeout 600 python bench.py --steps 5 --warmup 3 --profile-only > gpurun_out/spec_$v.json 2>&1
  python -c "import json;d=json.load(open('gpurun_out/spec_$v.json'));print('$v', round(d['value']), {k:round(v) for k,v in d['ops'].items()}, d['roofline']['kernel_ms_per_step'])"
done
