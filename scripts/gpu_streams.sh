for c in "c1" "c3 --scale 0.25 --shape TW" "c3 --scale 0.25 --shape RE" "c4 --shape COM" "c4 --shape LINE --scale 0.25"; do
  timeout 900 python bench.py --config $c --warmup 1 > gpurun_out/stream_$(echo $c | tr ' ' '_').json 2> gpurun_out/stream_err.txt
  tail -2 gpurun_out/stream_err.txt
  python -c "import json,sys;d=json.load(open('gpurun_out/stream_$(echo $c | tr ' ' '_').json'));print('$c', round(d['value']), d['ms_per_step'], d['ops'], d['fill_track']['min_after_mutation'], d['fill_track']['max'], d['resizes'], d['generator_seconds'])"
done
