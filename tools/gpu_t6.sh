O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > /dev/null 2>&1
timeout 1200 python -m pytest tests -m gpu -x -q > $O/pytest_t6.log 2>&1; echo "rc $?" >> $O/pytest_t6.log
timeout 300 python tools/panel_trace.py > $O/panel_trace6.log 2>&1
timeout 1500 python bench.py --n 65536 --b 64 --nb 2048 --mode 3xtf32 --steps 1 --warmup 1 --no-cpu-baseline --e2e-steps 0 --form-q-steps 0 --profile-steps 1 > $O/bench_cfg5.json 2> $O/bench_cfg5.err
