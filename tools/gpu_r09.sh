#!/bin/bash
# r07 A/B: GPU tests, the bench line, kxb cluster ablation, ncu launch list.
O=gpurun_out; mkdir -p $O; T=${1:-r07}
python -c "import __graft_entry__ as g; g.build()" > $O/build_$T.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_gpu_$T.log 2>&1; echo "rc $?" >> $O/pytest_gpu_$T.log
timeout 600 python bench.py --no-cpu-baseline --e2e-steps 0 > $O/bench_$T.json 2> $O/bench_$T.err
timeout 900 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$T.csv \
  python bench.py --steps 1 --warmup 0 --profile-steps 1 --e2e-steps 0 --no-cpu-baseline > $O/ncu_bench_$T.log 2>&1
python tools/launch_summary.py $O/launches_$T.csv > $O/launches_$T.txt 2>&1
echo done
