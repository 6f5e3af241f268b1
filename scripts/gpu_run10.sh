timeout 1500 python -m pytest tests -m gpu -x -q -k "not full_size" 2>&1 | tail -3
timeout 600 python bench.py --routed --steps 3 --warmup 2 --no-e2e > gpurun_out/bench_routed2.json 2> gpurun_out/bench_routed2.err; tail -3 gpurun_out/bench_routed2.err
python -c "import json;d=json.load(open('gpurun_out/bench_routed2.json'));print(round(d['value']), d['ms_per_step'], d['phase_ms_rank0'], d['roofline']['kernel_ms_per_step'], d['check'])"
