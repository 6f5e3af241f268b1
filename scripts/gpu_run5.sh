set -x
nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/gv scripts/gather_variants.cu
/tmp/gv
for B in 8 16 32; do
  timeout 600 python bench.py --steps 3 --warmup 2 --profile-only --bucket-slots $B > gpurun_out/bench_B$B.json 2>&1
  python -c "import json;d=json.load(open('gpurun_out/bench_B$B.json'));print($B, d['value'], d['ops'], d['roofline']['kernel_ms_per_step'], d['table'])"
done
