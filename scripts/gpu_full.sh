# Full measurement pass: tests, bench, ncu launch list + full captures, sanitizer.
R=${1:-r1}
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total,driver_version --format=csv > gpurun_out/gpu_$R.txt
timeout 1500 python -m pytest tests -m gpu -q 2>&1 | tail -5 > gpurun_out/pytest_gpu_$R.txt; cat gpurun_out/pytest_gpu_$R.txt
timeout 900 python bench.py > gpurun_out/bench_$R.json 2> gpurun_out/bench_$R.err; tail -2 gpurun_out/bench_$R.err; head -c 600 gpurun_out/bench_$R.json; echo
timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref_$R.json 2>&1; cat gpurun_out/bench_ref_$R.json | head -c 400; echo
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$R.csv python bench.py --steps 2 --warmup 1 --profile-only > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_upsert|k_find|k_delete|k_place" -c 4 -o gpurun_out/prof_$R python bench.py --steps 1 --warmup 0 --profile-only > gpurun_out/ncu_full_$R.log 2>&1; tail -2 gpurun_out/ncu_full_$R.log
timeout 900 compute-sanitizer --tool memcheck --error-exitcode 9 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/memcheck_$R.txt 2>&1; echo "memcheck rc=$?"; tail -3 gpurun_out/memcheck_$R.txt
ls -la gpurun_out
