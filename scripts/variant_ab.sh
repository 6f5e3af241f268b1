# A/B of prebuilt library variants in one GPU session: for each round, every
# variant runs `bench.py --profile-only` (C2) once, interleaved, so box-to-box
# and run-to-run drift hit all variants alike.
#   scripts/variant_ab.sh TAG ROUNDS lib1.so lib2.so ...
R=$1; N=$2; shift 2
mkdir -p gpurun_out
for i in $(seq 1 $N); do
  for lib in "$@"; do
    n=$(basename $lib .so)
    DYC_LIB=$lib timeout 600 python bench.py --profile-only --steps 5 --warmup 3 > gpurun_out/ab_${R}_${n}_$i.json 2>/dev/null
    python -c "import json,sys; x=json.loads(open(sys.argv[1]).read().strip().splitlines()[-1]); print(sys.argv[2], round(x['value']), {k: round(v,3) for k,v in x['roofline']['kernel_ms_per_step'].items()})" gpurun_out/ab_${R}_${n}_$i.json $n
  done
done
