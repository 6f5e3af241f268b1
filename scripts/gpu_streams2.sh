for c in "c1" "c3 --scale 0.25 --shape TW"; do
  timeout 900 python bench.py --config $c --warmup 1 > gpurun_out/stream2_$(echo $c | tr ' ' '_').json 2> gpurun_out/stream_err.txt
  tail -2 gpurun_out/stream_err.txt
  python -c "import json,sys;d=json.load(open('gpurun_out/stream2_$(echo $c | tr ' ' '_').json'));print('$c', round(d['value']), d['ms_per_step'], d['ops'], d['kernel_ms'], d['kernel_calls'], d['config']['batches'])"
done
