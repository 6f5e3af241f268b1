# Final pass after one-wave persistent grids for k_place / wide placement: full pass + wide config + C3-RE stream.
bash scripts/gpu_full.sh ${1:-r1zzz}
timeout 900 python bench.py --config wide > gpurun_out/wide_${1:-r1zzz}.json 2> gpurun_out/wide_err.txt; tail -2 gpurun_out/wide_err.txt
python -c "import json;d=json.load(open('gpurun_out/wide_${1:-r1zzz}.json'));print({m: round(v['step_mops']) for m,v in d['modes'].items()})"
for c in "c1" "c3 --scale 0.25 --shape TW" "c3 --shape RE" "c4 --shape LINE --scale 0.25" "c4 --shape COM"; do
  f=gpurun_out/stream_${1:-r1zzz}_$(echo $c | tr ' ' '_' | tr -d '-').json
  timeout 900 python bench.py --config $c --warmup 1 > $f 2> gpurun_out/stream_err.txt
  python -c "import json;d=json.load(open('$f'));print('$c', round(d['value']), d['ms_per_step'], d.get('kernel_ms'))"
done
