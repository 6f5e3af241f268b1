timeout 600 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/wide_launches.csv python bench.py --config wide --wide-modes lockfree_W1,grouped_W2 --steps 2 --warmup 1 > /dev/null 2>&1
python - <<'PY'
import csv, collections
rows = list(csv.reader(open('gpurun_out/wide_launches.csv')))
hdr = None; agg = collections.defaultdict(list)
for r in rows:
    if 'Kernel Name' in r: hdr = r; continue
    if hdr and len(r) == len(hdr):
        d = dict(zip(hdr, r))
        if d.get('Metric Name') == 'gpu__time_duration.sum':
            agg[d['Kernel Name'][:60]].append(float(d['Metric Value']))
for k, v in sorted(agg.items(), key=lambda x: -sum(x[1])):
    print(f"{k:60s} n={len(v):4d} total={sum(v)/1e6:.3f}ms mean={sum(v)/len(v)/1e3:.1f}us")
PY
