# Fused peer-memory routing: GPU tests (p2p + dist), then the routed C2 bench at N=1, NCCL router vs p2p router.
R=${1:-r1r}
timeout 900 python -X faulthandler -m pytest tests/test_gpu_p2p.py tests/test_gpu_dist.py -q -x 2>&1 | tail -15 > gpurun_out/pytest_p2p_$R.txt; cat gpurun_out/pytest_p2p_$R.txt
for m in "--routed" "--p2p"; do
  f=gpurun_out/bench_routed_${R}_$(echo $m | tr -d '-').json
  timeout 600 python bench.py $m --no-cpu-baseline --steps 5 > $f 2> gpurun_out/bench_routed_err.txt
  tail -3 gpurun_out/bench_routed_err.txt
  python -c "import json;d=json.load(open('$f'));print('$m', round(d['value']), d['ms_per_step'], d.get('phase_ms_rank0'), d['config'].get('routing'), d.get('check'))"
done
timeout 900 python bench.py --config c5 --p2p > gpurun_out/c5_p2p_$R.json 2> gpurun_out/c5.err; tail -3 gpurun_out/c5.err
python -c "import json;d=json.load(open('gpurun_out/c5_p2p_$R.json'));print(round(d['value']), d['phases'], d['check'], d['config']['routing'])"
