# C5 at N=1: local vs NCCL-routed vs p2p-routed, twice each (fill-time variance check).
R=${1:-r1t}
for rep in 1 2; do
for m in "" "--routed" "--p2p"; do
  f=gpurun_out/c5cmp_${R}_${rep}_$(echo "x$m" | tr -d '-').json
  timeout 600 python bench.py --config c5 $m > $f 2> gpurun_out/c5.err; tail -2 gpurun_out/c5.err
  python -c "import json;d=json.load(open('$f'));print('$m', round(d['value']), d['phases'], d['kernel_ms_rank0'], d['config']['routing'])"
done
done
