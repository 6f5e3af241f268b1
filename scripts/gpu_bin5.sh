timeout 900 python -m pytest tests/test_gpu_binned.py -x -q 2>&1 | tail -3
timeout 300 python scripts/bin_probe.py 1,0,0 1,19,0 2>&1 | tail -2
for v in bps4_u2 bps8_u1 bps2_u4 bps6_u1; do echo $v; DYC_LIB=variants/v_$v.so timeout 300 python scripts/bin_probe.py 1,19,0 2>&1 | tail -1; done
