#!/bin/bash
# Parameterised GPU runner (replaces the round-1 one-off lease scripts).
#   scripts/gpu_pass.sh TAG STEP [STEP ...]
# STEPs: tests | tests:<pytest -k expr> | bench | bench:<extra args> | ref | launches | ncu |
#        gather | sanitize | configs | smoke
# Everything lands in gpurun_out/ with TAG in the file name.
R=${1:?tag}; shift
mkdir -p gpurun_out
nvidia-smi --query-gpu=name,clocks.sm,clocks.max.sm,memory.total,driver_version --format=csv > gpurun_out/gpu_$R.txt
for step in "$@"; do
  case "$step" in
    tests) timeout 2400 python -m pytest tests -m gpu -q -x -p no:cacheprovider 2>&1 | tail -15 > gpurun_out/pytest_gpu_$R.txt; tail -3 gpurun_out/pytest_gpu_$R.txt ;;
    tests:*) timeout 2400 python -m pytest tests -m gpu -q -p no:cacheprovider -k "${step#tests:}" 2>&1 | tail -30 > gpurun_out/pytest_k_$R.txt; tail -5 gpurun_out/pytest_k_$R.txt ;;
    smoke) timeout 600 python -c "import __graft_entry__ as g; g.smoke()" 2>&1 | tail -2 ;;
    bench) timeout 1200 python bench.py > gpurun_out/bench_$R.json 2> gpurun_out/bench_$R.err; tail -2 gpurun_out/bench_$R.err; head -c 400 gpurun_out/bench_$R.json; echo ;;
    bench:*) a="${step#bench:}"; n=$(echo "$a" | tr -c 'a-zA-Z0-9' '_'); timeout 1800 python bench.py $a > gpurun_out/bench_${R}_$n.json 2> gpurun_out/bench_${R}_$n.err; tail -2 gpurun_out/bench_${R}_$n.err; head -c 300 gpurun_out/bench_${R}_$n.json; echo ;;
    ref) timeout 900 python bench.py --impl reference --steps 2 --warmup 1 > gpurun_out/bench_ref_$R.json 2>&1; head -c 300 gpurun_out/bench_ref_$R.json; echo ;;
    launches) timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file gpurun_out/launches_$R.csv python bench.py --steps 2 --warmup 1 --profile-only > /dev/null 2>&1; echo "launches rc=$?" ;;
    ncu) timeout 1500 ncu --set full --clock-control none --import-source on -k regex:"k_upsert|k_find|k_delete|k_place|k_st_" -c 20 -o gpurun_out/prof_$R python bench.py --steps 1 --warmup 0 --profile-only > gpurun_out/ncu_full_$R.log 2>&1; tail -2 gpurun_out/ncu_full_$R.log ;;
    gather) timeout 600 python scripts/gather_wall.py > gpurun_out/gather_$R.log 2>&1; tail -3 gpurun_out/gather_$R.log
            ;;
    sanitize)   # NOTE: compute-sanitizer was closed on the GPU pool during round 2 (r2n); kept for reference
      for tool in memcheck racecheck synccheck; do
        timeout 1500 compute-sanitizer --tool $tool --error-exitcode 9 python scripts/sanitize_streams.py > gpurun_out/${tool}_$R.txt 2>&1; echo "$tool rc=$?"; tail -2 gpurun_out/${tool}_$R.txt
      done ;;
    configs) for c in c1 "c3 --shape RE" "c3 --shape TW" "c4 --shape LINE" "c4 --shape COM"; do
               n=$(echo "$c" | tr -c 'a-zA-Z0-9' '_'); timeout 1200 python bench.py --config $c > gpurun_out/cfg_${R}_$n.json 2> gpurun_out/cfg_${R}_$n.err; head -c 250 gpurun_out/cfg_${R}_$n.json; echo; done ;;
    ablation)   # NEXT-4: placement rule x d x bucket width at C2, placement rule at C3-RE (x0.25)
      for pl in first_fit paper_weighted; do
        for d in 2 3 4 6 8; do
          timeout 900 python bench.py --placement $pl --d $d --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-rehash > gpurun_out/abl_${R}_${pl}_d$d.json 2> gpurun_out/abl_${R}_${pl}_d$d.err; head -c 200 gpurun_out/abl_${R}_${pl}_d$d.json; echo
        done
        timeout 900 python bench.py --placement $pl --bucket-slots 16 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-rehash > gpurun_out/abl_${R}_${pl}_B16.json 2>&1; head -c 200 gpurun_out/abl_${R}_${pl}_B16.json; echo
        timeout 900 python bench.py --placement $pl --bucket-slots 4 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-rehash > gpurun_out/abl_${R}_${pl}_B4.json 2>&1; head -c 200 gpurun_out/abl_${R}_${pl}_B4.json; echo
        timeout 900 python bench.py --config c3 --shape RE --scale 0.25 --placement $pl --no-cpu-baseline > gpurun_out/abl_${R}_${pl}_c3.json 2>&1; head -c 200 gpurun_out/abl_${R}_${pl}_c3.json; echo
      done ;;
    sweeps)     # NEXT-2: static fill factor at C2; r, alpha, beta, batch size at C3-TW x0.25 (Table tbl:parameters)
      for th in 0.7 0.75 0.8 0.85 0.9; do
        timeout 900 python bench.py --beta $th --alpha 0.1 --steps 3 --warmup 3 --no-e2e --no-cpu-baseline --no-rehash > gpurun_out/sw_${R}_theta$th.json 2>/dev/null; head -c 120 gpurun_out/sw_${R}_theta$th.json; echo
      done
      for a in "--r 0.1" "--r 0.2" "--r 0.3" "--r 0.5" "--alpha 0.2" "--alpha 0.4" "--beta 0.7" "--beta 0.9" "--batch 200000" "--batch 600000"; do
        n=$(echo "$a" | tr -c 'a-zA-Z0-9.' '_')
        timeout 900 python bench.py --config c3 --shape TW --scale 0.25 $a --no-cpu-baseline > gpurun_out/sw_${R}_c3$n.json 2>/dev/null; head -c 120 gpurun_out/sw_${R}_c3$n.json; echo
      done ;;
    *) echo "unknown step $step" ;;
  esac
done
ls gpurun_out | tail -40
