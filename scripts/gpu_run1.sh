set -x
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm --format=csv
python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -5
timeout 1200 python -m pytest tests -m gpu -x -q -k "not full_size" 2>&1 | tail -30
timeout 600 python bench.py --log2n 22 --steps 3 --warmup 3 --no-cpu-baseline 2>&1 | tail -5
