# NEXT-3 wide-key bench (all modes) + the C2 bench with the live-resize numbers.
R=${1:-wb}
timeout 900 python bench.py --config wide --steps 5 --warmup 3 > gpurun_out/wide_$R.json 2> gpurun_out/wide_$R.err; tail -3 gpurun_out/wide_$R.err
python -c "import json; d=json.load(open('gpurun_out/wide_$R.json')); [print(k, {a: round(b,3) if isinstance(b,float) else b for a,b in v.items()}) for k,v in d['modes'].items()]"
timeout 900 python bench.py --no-cpu-baseline --no-e2e > gpurun_out/bench_$R.json 2> gpurun_out/bench_$R.err; tail -3 gpurun_out/bench_$R.err
python -c "import json; d=json.load(open('gpurun_out/bench_$R.json')); print(d['value']); print({k: v for k, v in d['resize'].items() if 'live' in k or 'small' in k or 'alone' in k or 'sequential' in k})"
