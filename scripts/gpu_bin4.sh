timeout 900 python -m pytest tests/test_gpu_binned.py -x -q 2>&1 | tail -15
timeout 300 python scripts/bin_probe.py 0,0,0 1,0,0 1,19,0 1,18,0 2>&1 | tail -4
