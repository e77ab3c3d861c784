#!/bin/bash
# r11: final-state evidence of round 1 -- GPU tests, smoke, the default bench line (cpu_baseline + e2e),
# the reference arm, and the ncu launch list of the bench command
O=gpurun_out; mkdir -p $O; T=${1:-r11}
python -c "import __graft_entry__ as g; g.build()" > $O/build_$T.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_gpu_$T.log 2>&1; echo "rc $?" >> $O/pytest_gpu_$T.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_$T.log 2>&1; echo "rc $?" >> $O/smoke_$T.log
timeout 900 python bench.py > $O/bench_$T.json 2> $O/bench_$T.err
timeout 600 python bench.py --impl reference --steps 2 --warmup 0 > $O/bench_ref_$T.json 2> $O/bench_ref_$T.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$T.csv \
  python bench.py --steps 1 --warmup 0 --profile-steps 1 --e2e-steps 0 --no-cpu-baseline > $O/ncu_bench_$T.log 2>&1
python tools/launch_summary.py $O/launches_$T.csv > $O/launches_$T.txt 2>&1
gzip -f $O/launches_$T.csv
echo done
