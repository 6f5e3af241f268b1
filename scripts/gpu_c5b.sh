timeout 900 python bench.py --config c5 > gpurun_out/c5.json 2> gpurun_out/c5.err; tail -3 gpurun_out/c5.err
python -c "import json;d=json.load(open('gpurun_out/c5.json'));print(d['phases'], d['kernel_ms_rank0'], d['kernel_calls_rank0'])"
