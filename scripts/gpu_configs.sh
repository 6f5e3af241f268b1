# Every bench configuration once (short), to check the whole surface still runs.
for c in "c1" "c3 --scale 0.1" "c4 --scale 0.1" "c5 --c5-log2keys 28" "wide" ; do
  set -- $c
  timeout 600 python bench.py --config $c --steps 2 --warmup 1 --no-cpu-baseline --no-e2e > gpurun_out/cfg_$1.json 2> gpurun_out/cfg_$1.err
  echo "$c rc=$?"; head -c 400 gpurun_out/cfg_$1.json; echo; tail -2 gpurun_out/cfg_$1.err
done
timeout 600 python bench.py --routed --steps 2 --warmup 1 --no-cpu-baseline > gpurun_out/cfg_routed.json 2> gpurun_out/cfg_routed.err; echo "routed rc=$?"; head -c 400 gpurun_out/cfg_routed.json; echo
