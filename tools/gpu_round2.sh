#!/bin/bash
# Round trip: GPU tests + smoke, config-4 bench line, config-3 (3xTF32) bench line, ncu launch
# lists of both, full ncu captures of the dominant kernels of both modes.
TAG=${1:-r05}
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1
nvidia-smi > $O/smi_$TAG.txt 2>&1
if [ -z "$SKIP_TESTS" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q > $O/pytest_gpu_$TAG.log 2>&1; echo "pytest rc $?" >> $O/pytest_gpu_$TAG.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_$TAG.log 2>&1; echo "smoke rc $?" >> $O/smoke_$TAG.log
fi
timeout 900 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err
timeout 600 python bench.py --n 16384 --b 32 --nb 1024 --mode 3xtf32 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/bench_cfg3_$TAG.json 2> $O/bench_cfg3_$TAG.err
if [ -z "$SKIP_NCU" ]; then
  timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
    python bench.py --steps 1 --warmup 0 --profile-steps 1 --e2e-steps 0 --no-cpu-baseline > $O/ncu_bench_$TAG.log 2>&1
  python tools/launch_summary.py $O/launches_$TAG.csv > $O/launches_$TAG.txt 2>&1
  timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_cfg3_$TAG.csv \
    python bench.py --n 16384 --b 32 --nb 1024 --mode 3xtf32 --steps 1 --warmup 0 --profile-steps 1 --e2e-steps 0 --no-cpu-baseline > $O/ncu_bench_cfg3_$TAG.log 2>&1
  python tools/launch_summary.py $O/launches_cfg3_$TAG.csv > $O/launches_cfg3_$TAG.txt 2>&1
  for k in ${NCU_KERNELS-pass_tc_kernel gemm_tc_kernel panel_chol_kernel}; do
    skip=${NCU_SKIP:-300}; case $k in gemm_tc_kernel) skip=10;; esac
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s $skip -c 1 \
      -o $O/full_${k}_$TAG -f python tools/prof_run.py > $O/ncu_full_${k}_$TAG.log 2>&1
  done
  for k in ${NCU_KERNELS3-pass_tf32_kernel gemm_tc_kernel}; do
    skip=${NCU_SKIP:-150}; case $k in gemm_tc_kernel) skip=10;; esac
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s $skip -c 1 \
      -o $O/full3_${k}_$TAG -f python tools/prof_run.py --n 16384 --mode 3xtf32 > $O/ncu_full3_${k}_$TAG.log 2>&1
  done
fi
echo done
