# Full pass r1w (peer routing, block-aggregated downsize residuals, upsize occupancy): gpu tests, bench + reference arm, ncu launch list + full capture, memcheck.
bash scripts/gpu_full.sh r1w
