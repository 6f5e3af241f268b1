timeout 900 python -m pytest tests/test_gpu_binned.py -x -q 2>&1 | tail -15
timeout 300 python scripts/bin_probe.py 0,0,0 1,0,0 1,17,0 1,19,0 1,0,18 2>&1 | tail -6
for v in bps4_u2 bps3_u3 bps2_u2; do echo $v; DYC_LIB=variants/v_$v.so timeout 300 python scripts/bin_probe.py 1,0,0 2>&1 | tail -1; done
