# Full pass r1o (FFI + streaming resize kernels): gpu tests, bench + reference arm, ncu launch list + full capture, memcheck.
bash scripts/gpu_full.sh r1o
