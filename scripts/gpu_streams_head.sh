# Stream configs on the committed state (FFI + streaming resize): C1, C3 (TW, RE), C4 (LINE, COM), C5 at N=1.
R=${1:-r1q}
for c in "c1" "c3 --scale 0.25 --shape TW" "c3 --shape RE" "c4 --shape LINE --scale 0.25" "c4 --shape COM"; do
  f=gpurun_out/stream_${R}_$(echo $c | tr ' ' '_' | tr -d '-').json
  timeout 900 python bench.py --config $c --warmup 1 > $f 2> gpurun_out/stream_err.txt
  tail -2 gpurun_out/stream_err.txt
  python -c "import json,sys;d=json.load(open('$f'));print('$c', round(d['value']), d['ms_per_step'], d.get('ops'), d.get('kernel_ms'), d.get('kernel_calls'))"
done
timeout 900 python bench.py --config c5 > gpurun_out/c5_$R.json 2> gpurun_out/c5.err; tail -3 gpurun_out/c5.err
python -c "import json;d=json.load(open('gpurun_out/c5_$R.json'));print(round(d['value']), d['phases'], d['kernel_ms_rank0'], d['kernel_calls_rank0'])"
