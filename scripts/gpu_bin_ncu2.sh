export DYC_LIB=variants/v_bps4_u2.so
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/bin2_launches.csv python scripts/bin_probe.py 1,0,0 > /dev/null 2>&1
timeout 1200 ncu --set full --clock-control none --import-source on -k regex:"k_bin" -c 10 -o gpurun_out/bin2_prof python scripts/bin_probe.py 1,0,0 > gpurun_out/bin2_ncu.log 2>&1; tail -1 gpurun_out/bin2_ncu.log
