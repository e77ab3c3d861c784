#!/bin/bash
# config-5 parameters: b=64, nb=2048, 3xTF32 -- full-size parity at n=32768 and one bench step at n=65536 (1 GPU)
O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests/test_gpu_fullsize.py -q -x -s -k "64-2048" > $O/full5.log 2>&1; echo "rc $?" >> $O/full5.log
timeout 1500 python bench.py --n 65536 --b 64 --nb 2048 --mode 3xtf32 --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 --profile-steps 1 > $O/bench_cfg5.json 2> $O/bench_cfg5.err
