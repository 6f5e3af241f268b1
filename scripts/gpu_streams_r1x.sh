# Stream configs with the timed pass free of profiling scopes (kernel times from a separate replay); wide-key config refresh.
R=${1:-r1x}
for c in "c1" "c3 --scale 0.25 --shape TW" "c3 --shape RE" "c4 --shape LINE --scale 0.25" "c4 --shape COM"; do
  f=gpurun_out/stream_${R}_$(echo $c | tr ' ' '_' | tr -d '-').json
  timeout 900 python bench.py --config $c --warmup 1 > $f 2> gpurun_out/stream_err.txt
  tail -2 gpurun_out/stream_err.txt
  python -c "import json,sys;d=json.load(open('$f'));print('$c', round(d['value']), d['ms_per_step'], d.get('ops'), d.get('kernel_ms'), d.get('kernel_ms_source'))"
done
timeout 900 python bench.py --config wide > gpurun_out/wide_$R.json 2> gpurun_out/wide_err.txt; tail -2 gpurun_out/wide_err.txt
python -c "import json;d=json.load(open('gpurun_out/wide_$R.json'));print(json.dumps(d)[:1500])"
