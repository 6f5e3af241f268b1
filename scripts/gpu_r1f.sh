# Re-entry full pass: all gpu tests, bench (C2), reference arm, ncu launch list + full capture, wide bench, memcheck.
R=${1:-r1f}
bash scripts/gpu_full.sh $R
timeout 600 python bench.py --config wide --steps 5 --warmup 3 > gpurun_out/wide_$R.json 2> gpurun_out/wide_$R.err; tail -3 gpurun_out/wide_$R.err; head -c 1500 gpurun_out/wide_$R.json; echo
