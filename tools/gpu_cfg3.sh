#!/bin/bash
# 3xTF32 (config 3, n=16384 b=32 nb=1024): tensor-core path vs SIMT ablation, plus GPU tests.
O=gpurun_out; mkdir -p $O; T=${1:-r05}
python -c "import __graft_entry__ as g; g.build()" > $O/build_$T.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_gpu_$T.log 2>&1; echo "pytest rc $?" >> $O/pytest_gpu_$T.log
timeout 600 python bench.py --n 16384 --b 32 --nb 1024 --mode 3xtf32 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 > $O/bench_cfg3_$T.json 2> $O/bench_cfg3_$T.err
SBR_TF32_TC=0 timeout 600 python bench.py --n 16384 --b 32 --nb 1024 --mode 3xtf32 --steps 2 --warmup 1 --no-cpu-baseline --e2e-steps 0 --profile-steps 1 > $O/bench_cfg3_simt_$T.json 2> $O/bench_cfg3_simt_$T.err
echo done
