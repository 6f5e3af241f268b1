# NEXT-3 wide-key table: parity tests (+ live-resize tests) on the GPU.
R=${1:-wide}
timeout 1200 python -m pytest tests/test_gpu_wide.py -x -q 2>&1 | tail -30 > gpurun_out/pytest_wide_$R.txt; cat gpurun_out/pytest_wide_$R.txt
