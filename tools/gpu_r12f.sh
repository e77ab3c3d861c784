#!/bin/bash
# CholeskyQR: LU overlapped with CTA 0's Gram: GPU tests, config-4 A/B (SBR_PANEL_LU=serial), chain trace
O=gpurun_out; mkdir -p $O; T=${1:-r12f}
timeout 600 python -m pytest tests -m gpu -x -q > $O/pytest_gpu_$T.log 2>&1; echo "rc $?" >> $O/pytest_gpu_$T.log
timeout 300 python -c "import __graft_entry__ as g; g.smoke()" > $O/smoke_$T.log 2>&1; echo "rc $?" >> $O/smoke_$T.log
timeout 300 python bench.py --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 > $O/bench_ov_$T.json 2> $O/bench_ov_$T.err
SBR_PANEL_LU=serial timeout 300 python bench.py --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 > $O/bench_se_$T.json 2> $O/bench_se_$T.err
timeout 300 python tools/panel_chain_trace.py > $O/panel_chain_trace_$T.txt 2>&1
echo done
