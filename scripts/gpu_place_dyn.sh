# k_place with dynamic chunk distribution: full GPU tests, C2 bench, stream configs.
R=${1:-r1v}
timeout 1500 python -X faulthandler -m pytest tests -m gpu -q -x 2>&1 | tail -4 > gpurun_out/pytest_gpu_$R.txt; cat gpurun_out/pytest_gpu_$R.txt
timeout 600 python bench.py --no-rehash --steps 5 > gpurun_out/bench_$R.json 2>/dev/null
python -c "import json;d=json.load(open('gpurun_out/bench_$R.json'));r=d['roofline'];print('c2', round(d['value']), r['kernel_ms_per_step'], r.get('frac_of_access_ceiling'), d['table'])"
for c in "c1" "c3 --scale 0.25 --shape TW" "c3 --shape RE" "c4 --shape COM"; do
  f=gpurun_out/stream_${R}_$(echo $c | tr ' ' '_' | tr -d '-').json
  timeout 900 python bench.py --config $c --warmup 1 > $f 2> gpurun_out/stream_err.txt
  tail -2 gpurun_out/stream_err.txt
  python -c "import json,sys;d=json.load(open('$f'));print('$c', round(d['value']), d['ms_per_step'], d.get('ops'), d.get('kernel_ms'), d.get('kernel_calls'))"
done
