#!/bin/bash
# One GPU round trip (run from the repo root under gpurun):
#   bash tools/gpu_round.sh TAG [steps...]
# steps (default: build tests smoke bench):
#   build        compile libsbr
#   tests        pytest -m gpu (PYTEST_ARGS to narrow, e.g. "-k table3")
#   smoke        __graft_entry__.smoke()
#   bench        default bench line (config 4)               -> bench_TAG.json
#   cfg2|cfg3|cfg5  bench lines of configs 2, 3 and config-5 parameters
#   ref          bench.py --impl reference
#   launches     ncu launch list of one bench step            -> launches_TAG.{csv,txt}
#   ncu          ncu --set full of NCU_KERNELS (regex list; NCU_SKIP launches skipped)
#   sanitize     compute-sanitizer racecheck/synccheck on config 1
# Everything lands in gpurun_out/ (copy what is to be judged into profiles/).
TAG=${1:-rX}; shift
STEPS=${*:-build tests smoke bench}
O=gpurun_out
mkdir -p $O
for s in $STEPS; do
  case $s in
    build) python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1; echo "build rc $?" >> $O/build_$TAG.log;;
    tests) timeout ${TEST_TIMEOUT:-1800} python -m pytest tests -m gpu -q -s -x $PYTEST_ARGS > $O/pytest_gpu_$TAG.log 2>&1
           echo "pytest rc $?" >> $O/pytest_gpu_$TAG.log;;
    smoke) timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_$TAG.log 2>&1; echo "smoke rc $?" >> $O/smoke_$TAG.log;;
    bench) timeout 900 python bench.py $BENCH_ARGS > $O/bench_$TAG.json 2> $O/bench_$TAG.err;;
    cfg2) timeout 600 python bench.py --n 4096 --b 32 --nb 256 --mode fp16 --input geo --steps 20 --warmup 5 \
            --form-q-steps 0 > $O/bench_cfg2_$TAG.json 2> $O/bench_cfg2_$TAG.err;;
    cfg3) timeout 600 python bench.py --n 16384 --b 32 --nb 1024 --mode 3xtf32 --steps 5 --warmup 3 \
            --form-q-steps 0 > $O/bench_cfg3_$TAG.json 2> $O/bench_cfg3_$TAG.err;;
    cfg5) timeout 1500 python bench.py --n 65536 --b 64 --nb 2048 --mode 3xtf32 --input geo --steps 2 --warmup 1 \
            --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 --profile-steps 1 > $O/bench_cfg5_$TAG.json 2> $O/bench_cfg5_$TAG.err;;
    ref) timeout 900 python bench.py --impl reference --steps ${REF_STEPS:-5} --warmup 1 > $O/bench_ref_$TAG.json 2> $O/bench_ref_$TAG.err;;
    launches)
      timeout 1500 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
        python tools/prof_run.py $PROF_ARGS > $O/ncu_launches_$TAG.log 2>&1
      python tools/launch_summary.py $O/launches_$TAG.csv > $O/launches_$TAG.txt 2>&1;;
    ncu)
      for k in ${NCU_KERNELS:-pass_tc_kernel}; do
        kn=$(echo "$k" | tr -c 'A-Za-z0-9_\n' '_')
        sk=${NCU_SKIP:-300}; case $k in *gemm_tc*|*chain*|*s2_*) sk=${NCU_SKIP_GEMM:-0};; esac
        timeout 900 ncu --set full --clock-control none --import-source on --kernel-name-base ${NCU_BASE:-function} \
          -k "regex:$k" -s $sk -c 1 -o $O/full_${kn}_$TAG -f python tools/prof_run.py $PROF_ARGS > $O/ncu_full_${kn}_$TAG.log 2>&1
        python tools/ncu_summary.py $O/full_${kn}_$TAG.ncu-rep > $O/ncu_full_${kn}_$TAG.txt 2>&1
      done;;
    sanitize)
      for tool in racecheck synccheck memcheck; do
        timeout 900 compute-sanitizer --tool $tool --print-limit 20 python -c "import __graft_entry__ as g; g.smoke()" \
          > $O/sanitize_${tool}_$TAG.log 2>&1; echo "rc $?" >> $O/sanitize_${tool}_$TAG.log
      done;;
  esac
done
echo done
