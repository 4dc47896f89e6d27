# full GPU suite then a bench line
timeout -s KILL 1200 python -m pytest tests -m gpu -q --timeout 300 -x 2>&1 | tail -15
timeout -s KILL 1200 python bench.py "$@" > gpurun_out/bench.json 2> gpurun_out/bench.err; echo "bench rc=$?"
tail -3 gpurun_out/bench.err
