R=${1:-w2}
timeout 1200 python -m pytest tests/test_gpu_wide.py tests/test_gpu_live_resize.py -x -q 2>&1 | tail -5; 
bash scripts/gpu_wide_bench.sh $R
