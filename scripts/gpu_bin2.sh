timeout 900 python -m pytest tests/test_gpu_binned.py -x -q 2>&1 | tail -4
timeout 600 python scripts/bin_probe.py 1,0,0 2,0,0 2,17,0 2,19,0 2,15,0 2,0,16 2>&1 | tail -12
