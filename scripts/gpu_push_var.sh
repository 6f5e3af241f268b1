# push-kernel variants: routed p2p C2 step, per-phase times.
R=${1:-r1zb}
for v in default build/var_*.so; do
  if [ "$v" = default ]; then unset DYC_LIB; else export DYC_LIB=$v; fi
  timeout 600 python bench.py --p2p --no-cpu-baseline --no-e2e --steps 3 > gpurun_out/push_${R}_$(basename $v .so).json 2>/dev/null
  python -c "import json;d=json.load(open('gpurun_out/push_${R}_$(basename $v .so).json'));print('$v', round(d['value']), d['ms_per_step'], d.get('phase_ms_rank0'))"
done
unset DYC_LIB
timeout 800 ncu --metrics gpu__time_duration.sum --clock-control none -k regex:"k_route_push" -c 3 --csv --log-file gpurun_out/push_dev_$R.csv env DYC_LIB=build/var_devatomic.so python bench.py --p2p --steps 1 --warmup 0 --no-cpu-baseline --no-e2e > /dev/null 2>&1
grep -o '"gpu__time_duration.sum","[^"]*","[0-9.,]*"' gpurun_out/push_dev_$R.csv | head -3
