for u in 1 2 4; do
  if [ $u = 4 ]; then L=paper_conf_icde_lizlhs21_b200/libdyc.so; else L=paper_conf_icde_lizlhs21_b200/libdyc_u$u.so; fi
  DYC_LIB=$L timeout 600 python bench.py --config wide --wide-modes lockfree_W1,grouped_W2,voter_W2 --steps 5 --warmup 3 > gpurun_out/wideu_$u.json 2>/dev/null
  echo "U=$u"; python -c "import json; d=json.load(open('gpurun_out/wideu_$u.json')); [print(k, {a: round(b,3) if isinstance(b,float) else b for a,b in v.items() if 'mops' in a or 'ms' in a}) for k,v in d['modes'].items()]"
done
