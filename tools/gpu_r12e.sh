#!/bin/bash
# evict_first in the 3xTF32 pass: full GPU tests, config-3 A/B (SBR_TF32_L2=normal), config-4 bench
O=gpurun_out; mkdir -p $O; T=${1:-r12e}
timeout 600 python -m pytest tests -m gpu -x -q > $O/pytest_gpu_$T.log 2>&1; echo "rc $?" >> $O/pytest_gpu_$T.log
A="--n 16384 --b 32 --nb 1024 --mode 3xtf32 --no-cpu-baseline --e2e-steps 0 --form-q-steps 0"
timeout 300 python bench.py $A > $O/bench_cfg3_ef_$T.json 2> $O/bench_cfg3_ef_$T.err
SBR_TF32_L2=normal timeout 300 python bench.py $A > $O/bench_cfg3_en_$T.json 2> $O/bench_cfg3_en_$T.err
timeout 300 python bench.py --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 > $O/bench_$T.json 2> $O/bench_$T.err
echo done
