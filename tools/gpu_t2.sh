O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_t2.log 2>&1
timeout 600 python -m pytest tests/test_gpu_formq.py -q -x -s 2>&1 | grep -E "form_q|passed|failed|Error|assert" > $O/formq.log
timeout 600 python -m pytest tests/test_gpu_parity.py tests/test_gpu_fullsize.py -q -x -k "3xtf32" 2>&1 | tail -3 > $O/par3.log
timeout 600 python bench.py --n 16384 --b 32 --nb 1024 --mode 3xtf32 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 0 > $O/bench_cfg3_t2.json 2> $O/bench_cfg3_t2.err
timeout 300 python tools/panel_trace.py > $O/panel_trace.log 2>&1
