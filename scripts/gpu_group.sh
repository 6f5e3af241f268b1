# Warp-aggregated ranking in the grouping kernels: all GPU tests, routed C2 (NCCL / p2p), C4 mixed streams, launch list of the route kernels.
R=${1:-r1za}
timeout 1500 python -m pytest tests -m gpu -q -x 2>&1 | tail -3 > gpurun_out/pytest_gpu_$R.txt; cat gpurun_out/pytest_gpu_$R.txt
for m in "--routed" "--p2p"; do
  f=gpurun_out/bench_routed_${R}_$(echo $m | tr -d '-').json
  timeout 600 python bench.py $m --no-cpu-baseline --no-e2e --steps 5 > $f 2> gpurun_out/err.txt; tail -2 gpurun_out/err.txt
  python -c "import json;d=json.load(open('$f'));print('$m', round(d['value']), d['ms_per_step'], d.get('phase_ms_rank0'))"
done
for c in "c4 --shape LINE --scale 0.25" "c4 --shape COM"; do
  f=gpurun_out/stream_${R}_$(echo $c | tr ' ' '_' | tr -d '-').json
  timeout 900 python bench.py --config $c --warmup 1 > $f 2> gpurun_out/err.txt; tail -2 gpurun_out/err.txt
  python -c "import json;d=json.load(open('$f'));print('$c', round(d['value']), d['ms_per_step'], d.get('kernel_ms'))"
done
timeout 800 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_route|k_group" --csv --log-file gpurun_out/launches_route_$R.csv python bench.py --p2p --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
timeout 800 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_route|k_group" --csv --log-file gpurun_out/launches_nccl_$R.csv python bench.py --routed --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
ls -la gpurun_out | grep $R
