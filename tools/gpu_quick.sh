python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 600 python -m pytest tests -m gpu -x -q -k "ws_equals or c1 or heavy or fuzz or full_frame or band" > gpurun_out/gpu_tests.log 2>&1
timeout 300 python bench.py --no-e2e --no-cpu-baseline > gpurun_out/bench.json 2> gpurun_out/bench.err
tail -5 gpurun_out/gpu_tests.log
