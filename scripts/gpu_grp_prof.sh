timeout 600 ncu --metrics gpu__time_duration.sum,dram__bytes_read.sum,dram__bytes_write.sum --csv --log-file gpurun_out/ncu_grp.csv python bench.py --steps 1 --warmup 0 --profile-only > /dev/null 2>&1
python3 - <<'PY'
import csv
rows=list(csv.reader(open('gpurun_out/ncu_grp.csv')))
i=[k for k,r in enumerate(rows) if r and r[0]=='ID'][0]
hdr=rows[i]; ki=hdr.index('Kernel Name'); mi=hdr.index('Metric Name'); vi=hdr.index('Metric Value'); ii=hdr.index('ID'); ui=hdr.index('Metric Unit')
d={}
for r in rows[i+1:]:
    d.setdefault((int(r[ii]),r[ki][:40]),{})[r[mi].split('__')[1]]=r[vi]+r[ui]
for k,m in sorted(d.items()):
    if 'dyc' in k[1] or 'k_' in k[1]: print(k, m)
PY
