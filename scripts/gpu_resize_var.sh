# Resize-kernel unroll variants (C2 step, kernel times) + C5 fill with allocation timing (local, twice).
R=${1:-r1u}
bash scripts/gpu_variants.sh $R
for rep in 1 2; do
  timeout 600 python bench.py --config c5 > gpurun_out/c5alloc_${R}_$rep.json 2> gpurun_out/c5.err; tail -2 gpurun_out/c5.err
  python -c "import json;d=json.load(open('gpurun_out/c5alloc_${R}_$rep.json'));print(round(d['value']), d['phases'], d['shard0'])"
done
