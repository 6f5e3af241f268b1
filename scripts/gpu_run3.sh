set -x
python scripts/gather_sweep.py 2>&1 | tail -12
for g in 32 64 128; do
  timeout 600 python bench.py --steps 3 --warmup 2 --profile-only --l2-fetch $g > gpurun_out/bench_l2_$g.json 2>&1
  python -c "import json;d=json.load(open('gpurun_out/bench_l2_$g.json'));print($g, d['ops'], d['roofline']['kernel_ms_per_step'], d['roofline']['random_32B_gather_gbs'])"
done
for g in 32 128; do
timeout 600 ncu --metrics gpu__time_duration.sum,dram__sectors_read.sum,dram__sectors_write.sum,lts__t_sectors_srcunit_tex_op_read.sum,lts__t_requests_srcunit_tex_op_read.sum -k regex:"k_" --csv --log-file gpurun_out/ncu_l2_$g.csv python bench.py --steps 1 --warmup 0 --profile-only --l2-fetch $g > /dev/null 2>&1
done
ls gpurun_out
