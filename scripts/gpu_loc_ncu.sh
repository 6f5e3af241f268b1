timeout 900 ncu --metrics gpu__time_duration.sum,dram__sectors_read.sum,dram__sectors_write.sum,lts__t_sector_hit_rate.pct,lts__t_requests_srcunit_tex_op_read.sum,lts__t_sector_op_read_hit_rate.pct,lts__t_sector_op_atom_hit_rate.pct -k regex:"k_upsert|k_place" --csv --log-file gpurun_out/ncu_loc.csv python scripts/locality_ncu.py > gpurun_out/loc_ncu.log 2>&1
python3 - <<'PY'
import csv
rows=list(csv.reader(open('gpurun_out/ncu_loc.csv')))
i=[k for k,r in enumerate(rows) if r and r[0]=='ID'][0]
hdr=rows[i]; ki=hdr.index('Kernel Name'); mi=hdr.index('Metric Name'); vi=hdr.index('Metric Value'); ii=hdr.index('ID')
d={}
for r in rows[i+1:]:
    d.setdefault((int(r[ii]),r[ki][:14]),{})[r[mi].split('__')[1]]=r[vi]
for k,m in sorted(d.items()): print(k, m)
PY
tail -3 gpurun_out/loc_ncu.log
