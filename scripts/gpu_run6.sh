nvcc -O3 -gencode arch=compute_100a,code=sm_100a -o /tmp/gv scripts/gather_variants.cu
/tmp/gv
timeout 600 ncu --metrics gpu__time_duration.sum,dram__sectors_read.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_requests_srcunit_tex_op_read.sum --csv --log-file gpurun_out/ncu_variants2.csv -k regex:"g<1[0-4]>" -c 15 /tmp/gv > /dev/null 2>&1
python3 - <<'PY'
import csv
rows=list(csv.reader(open('gpurun_out/ncu_variants2.csv')))
i=[k for k,r in enumerate(rows) if r and r[0]=='ID'][0]
hdr=rows[i]; ki=hdr.index('Kernel Name'); mi=hdr.index('Metric Name'); vi=hdr.index('Metric Value'); ii=hdr.index('ID')
d={}
for r in rows[i+1:]:
    d.setdefault((int(r[ii]),r[ki][:12]),{})[r[mi].split('__')[1]]=r[vi]
for k,m in sorted(d.items()): print(k, m)
PY
