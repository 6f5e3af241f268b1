# Final pass of the session (after the grouping/push changes): gpu tests, bench + reference arm, ncu launch list + full capture, memcheck; routed p2p launch list.
bash scripts/gpu_full.sh r1zz
timeout 800 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --clock-control none -k regex:"k_route" --csv --log-file gpurun_out/launches_p2p_r1zz.csv python bench.py --p2p --steps 1 --warmup 1 --no-cpu-baseline --no-e2e > /dev/null 2>&1
