timeout 1500 python -m pytest tests -m gpu -x -q -k "not full_size" 2>&1 | tail -3
timeout 900 python bench.py --config c5 > gpurun_out/c5.json 2> gpurun_out/c5.err; tail -3 gpurun_out/c5.err; head -c 2000 gpurun_out/c5.json; echo
timeout 900 python bench.py --config c5 --routed > gpurun_out/c5r.json 2> gpurun_out/c5r.err; tail -3 gpurun_out/c5r.err; head -c 800 gpurun_out/c5r.json; echo
