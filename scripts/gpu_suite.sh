# Full GPU test suite with a verbose log (finds the test a crash happens in).
R=${1:-r1}
timeout 600 python -m pytest tests/test_gpu_ffi.py -q -x 2>&1 | tail -25 > gpurun_out/pytest_ffi_$R.txt; tail -3 gpurun_out/pytest_ffi_$R.txt
timeout 1500 python -X faulthandler -m pytest tests -m gpu -v -x -p no:cacheprovider > gpurun_out/pytest_gpu_full_$R.txt 2>&1; echo "rc=$?"
grep -n "PASSED\|FAILED\|ERROR" gpurun_out/pytest_gpu_full_$R.txt | tail -3; grep -n -B2 -A12 "Fatal Python\|Segmentation" gpurun_out/pytest_gpu_full_$R.txt | head -60; tail -3 gpurun_out/pytest_gpu_full_$R.txt
