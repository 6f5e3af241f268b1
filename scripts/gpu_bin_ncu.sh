timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/bin_launches.csv python scripts/bin_probe.py 2,0,0 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_bin" -c 12 -o gpurun_out/bin_prof python scripts/bin_probe.py 2,0,0 > gpurun_out/bin_ncu.log 2>&1; tail -2 gpurun_out/bin_ncu.log
