#!/bin/bash
# evict_first OA stream in the fp16 pass: pass parity tests, then config-4 bench A/B (SBR_PASS_EXPER=4 = old
# evict_normal policy) and the panel chain trace
O=gpurun_out; mkdir -p $O; T=${1:-r12d}
timeout 400 python -m pytest tests -m gpu -x -q -k "pass or smoke or fp16" > $O/pytest_pass_$T.log 2>&1; echo "rc $?" >> $O/pytest_pass_$T.log
timeout 400 python bench.py --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 > $O/bench_ef_$T.json 2> $O/bench_ef_$T.err
SBR_PASS_EXPER=4 timeout 400 python bench.py --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 > $O/bench_en_$T.json 2> $O/bench_en_$T.err
timeout 300 python tools/panel_chain_trace.py > $O/panel_chain_trace_$T.txt 2>&1
echo done
