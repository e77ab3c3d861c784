#!/bin/bash
# One GPU round trip: GPU tests, the bench line, the ncu launch list of the bench command and
# full ncu captures of the dominant kernels.  Usage (from the repo root, under gpurun):
#   bash tools/gpu_round.sh [tag]
TAG=${1:-r01}
O=gpurun_out
mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_$TAG.log 2>&1
nvidia-smi > $O/smi_$TAG.txt 2>&1
if [ -z "$SKIP_TESTS" ]; then
  timeout 1200 python -m pytest tests -m gpu -x -q > $O/pytest_gpu_$TAG.log 2>&1; echo "pytest rc $?" >> $O/pytest_gpu_$TAG.log
  timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_$TAG.log 2>&1; echo "smoke rc $?" >> $O/smoke_$TAG.log
fi
timeout 900 python bench.py > $O/bench_$TAG.json 2> $O/bench_$TAG.err
if [ -z "$SKIP_NCU" ]; then
  timeout 1200 ncu --metrics gpu__time_duration.sum --clock-control none --csv --log-file $O/launches_$TAG.csv \
    python bench.py --steps 1 --warmup 0 --profile-steps 1 --e2e-steps 0 --no-cpu-baseline > $O/ncu_bench_$TAG.log 2>&1
  python tools/launch_summary.py $O/launches_$TAG.csv > $O/launches_$TAG.txt 2>&1
  for k in ${NCU_KERNELS-pass_tc_kernel gemm_tc_kernel panel_chol_kernel skinny_nn_kernel kxb_kernel postpass_kernel skinny_tn_kernel}; do
    skip=${NCU_SKIP:-300}; case $k in gemm_tc_kernel) skip=10;; esac
    timeout 600 ncu --set full --clock-control none --import-source on -k regex:$k -s $skip -c 1 \
      -o $O/full_${k}_$TAG -f python tools/prof_run.py > $O/ncu_full_${k}_$TAG.log 2>&1
  done
fi
echo done
