# Final pass of the round: d=2 sweep point, full measurement pass, racecheck on smoke.
R=${1:-r1d}
timeout 600 python bench.py --d 2 --steps 3 --warmup 3 --profile-only --no-cpu-baseline --no-e2e > gpurun_out/sw_d2.json 2> gpurun_out/sw_d2.err; head -c 400 gpurun_out/sw_d2.json; echo
bash scripts/gpu_full.sh $R
timeout 900 compute-sanitizer --tool racecheck --error-exitcode 9 python -c "import __graft_entry__ as g; g.smoke()" > gpurun_out/racecheck_$R.txt 2>&1; echo "racecheck rc=$?"; tail -3 gpurun_out/racecheck_$R.txt
