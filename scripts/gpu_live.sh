# NEXT-1 (resize under live traffic): parity tests + the bench's live-resize numbers.
R=${1:-live}
timeout 900 python -m pytest tests/test_gpu_live_resize.py -x -q 2>&1 | tail -25 > gpurun_out/pytest_live_$R.txt; cat gpurun_out/pytest_live_$R.txt
timeout 1200 python -m pytest tests -m gpu -x -q 2>&1 | tail -5 > gpurun_out/pytest_gpu_$R.txt; cat gpurun_out/pytest_gpu_$R.txt
timeout 900 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_$R.json 2> gpurun_out/bench_$R.err; tail -3 gpurun_out/bench_$R.err
python -c "import json; d=json.load(open('gpurun_out/bench_$R.json')); print(d['value'], d['resize'])"
