# Bench the default library and every build/var_*.so (C2, kernel times per step).
R=${1:-r1}
for v in default build/var_*.so; do
  if [ "$v" = default ]; then unset DYC_LIB; else export DYC_LIB=$v; fi
  timeout 600 python bench.py --no-rehash --steps 3 > gpurun_out/bench_${R}_$(basename $v .so).json 2>/dev/null
  python -c "
import json; d=json.load(open('gpurun_out/bench_${R}_$(basename $v .so).json')); r=d['roofline']; print('$v', round(d['value']), r['kernel_ms_per_step'], r['frac_of_access_ceiling'])"
done
