nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/wv scripts/write_variants.cu
/tmp/wv
timeout 600 ncu --metrics gpu__time_duration.sum,dram__sectors_read.sum,dram__sectors_write.sum --csv --log-file gpurun_out/ncu_writes.csv -c 30 /tmp/wv > /dev/null 2>&1
python3 - <<'PY'
import csv
rows=list(csv.reader(open('gpurun_out/ncu_writes.csv')))
i=[k for k,r in enumerate(rows) if r and r[0]=='ID'][0]
hdr=rows[i]; ki=hdr.index('Kernel Name'); mi=hdr.index('Metric Name'); vi=hdr.index('Metric Value'); ii=hdr.index('ID')
d={}
for r in rows[i+1:]:
    d.setdefault((int(r[ii]),r[ki][:8]),{})[r[mi].split('__')[1]]=r[vi]
for k,m in sorted(d.items()):
    if k[0] % 3 == 2: print(k, m)
PY
