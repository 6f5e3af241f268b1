# Final full pass r1z: gpu tests (seeded parity, p2p), bench + reference arm, ncu launch list + full capture, memcheck.
bash scripts/gpu_full.sh r1z
