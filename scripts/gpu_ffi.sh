# FFI (first-choice-full invariant) pass: new tests, full gpu suite, bench default + register-cap variant.
R=${1:-r1j}
timeout 600 python -m pytest tests/test_gpu_ffi.py -q -x 2>&1 | tail -25 > gpurun_out/pytest_ffi_$R.txt; cat gpurun_out/pytest_ffi_$R.txt
timeout 1500 python -X faulthandler -m pytest tests -m gpu -q -x 2>&1 | tail -30 > gpurun_out/pytest_gpu_$R.txt; cat gpurun_out/pytest_gpu_$R.txt
timeout 900 python bench.py --no-rehash > gpurun_out/bench_$R.json 2> gpurun_out/bench_$R.err; tail -2 gpurun_out/bench_$R.err
python - gpurun_out/bench_$R.json <<'PY'
import json,sys
d=json.load(open(sys.argv[1]))
r=d["roofline"]
print("value",d["value"],"phase",{k:round(v,3) for k,v in d["phase_ms"].items()})
print("kern",r["kernel_ms_per_step"],"acc_frac",r["frac_of_access_ceiling"],"model",r["model"])
PY
for v in build/var_*.so; do echo "== $v"; DYC_LIB=$v timeout 900 python bench.py --no-rehash --steps 3 > gpurun_out/bench_${R}_$(basename $v .so).json 2>/dev/null; python -c "
import json; d=json.load(open('gpurun_out/bench_${R}_$(basename $v .so).json')); print(d['value'], d['roofline']['kernel_ms_per_step'])"; done
