O=gpurun_out; mkdir -p $O
python -c "import __graft_entry__ as g; g.build()" > $O/build_t3.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > $O/pytest_t3.log 2>&1; echo "rc $?" >> $O/pytest_t3.log
timeout 600 python bench.py --n 16384 --b 32 --nb 1024 --mode 3xtf32 --steps 3 --warmup 3 --no-cpu-baseline --e2e-steps 1 --form-q-steps 2 > $O/bench_cfg3_t3.json 2> $O/bench_cfg3_t3.err
