timeout 600 ncu --metrics gpu__time_duration.sum --csv --log-file gpurun_out/ncu_routed.csv python bench.py --routed --steps 1 --warmup 0 --no-e2e --profile-only > /dev/null 2>&1
python3 - <<'PY'
import csv, collections
rows=list(csv.reader(open('gpurun_out/ncu_routed.csv')))
i=[k for k,r in enumerate(rows) if r and r[0]=='ID'][0]
hdr=rows[i]; ki=hdr.index('Kernel Name'); vi=hdr.index('Metric Value'); ii=hdr.index('ID')
L=[(int(r[ii]), r[ki][:60], float(r[vi].replace(',',''))/1e6) for r in rows[i+1:]]
# print the last 60 launches (the timed step)
for x in L[-70:]: print(x)
PY
