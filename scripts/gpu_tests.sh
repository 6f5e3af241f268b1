timeout 1500 python -m pytest tests -m gpu -x -q -k "not full_size" 2>&1 | tail -15
