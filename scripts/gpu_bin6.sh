timeout 900 python -m pytest tests/test_gpu_binned.py -x -q 2>&1 | tail -3
timeout 300 python scripts/bin_probe.py 0,0,0 1,19,0 2>&1 | tail -2
for v in bps3_u2 bps2_u2 bps3_u1 bps4_u1; do echo $v; DYC_LIB=variants/v_$v.so timeout 300 python scripts/bin_probe.py 1,19,0 2>&1 | tail -1; done
