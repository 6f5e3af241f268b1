# Full pass r1i: all gpu tests, bench (C2) + reference arm, ncu launch list + full capture, memcheck.
bash scripts/gpu_full.sh r1i
