#!/bin/bash
# r10: GPU tests, bench, launch list, ncu captures of LATE (small-M) skinny_nn / pass launches
O=gpurun_out; mkdir -p $O; T=${1:-r10}
python -c "import __graft_entry__ as g; g.build()" > $O/build_$T.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_gpu_$T.log 2>&1; echo "rc $?" >> $O/pytest_gpu_$T.log
timeout 600 python bench.py --no-cpu-baseline --e2e-steps 0 > $O/bench_$T.json 2> $O/bench_$T.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$T.csv \
  python bench.py --steps 1 --warmup 0 --profile-steps 1 --e2e-steps 0 --no-cpu-baseline > $O/ncu_bench_$T.log 2>&1
python tools/launch_summary.py $O/launches_$T.csv > $O/launches_$T.txt 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:skinny_nn -s 1960 -c 1 \
  -o $O/full_skinny_nn_late_$T -f python tools/prof_run.py > $O/ncu_full_nn_late_$T.log 2>&1
timeout 600 ncu --set full --clock-control none --import-source on -k regex:pass_tc -s 1000 -c 1 \
  -o $O/full_pass_late_$T -f python tools/prof_run.py > $O/ncu_full_pass_late_$T.log 2>&1
echo done
