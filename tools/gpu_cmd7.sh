python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_r07.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/pytest_gpu_r07.log 2>&1; echo "rc $?" >> gpurun_out/pytest_gpu_r07.log
timeout 600 python bench.py --no-cpu-baseline --e2e-steps 0 > gpurun_out/bench_r07.json 2> gpurun_out/bench_r07.err
timeout 600 python bench.py --no-cpu-baseline --e2e-steps 0 --n 16384 --mode 3xtf32 --steps 3 > gpurun_out/bench_r07_cfg3.json 2>> gpurun_out/bench_r07.err
timeout 600 python bench.py --no-cpu-baseline --e2e-steps 0 --n 4096 --nb 256 --steps 5 > gpurun_out/bench_r07_cfg2.json 2>> gpurun_out/bench_r07.err
