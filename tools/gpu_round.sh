python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build.log 2>&1
timeout 900 python -m pytest tests -m gpu -x -q > gpurun_out/gpu_tests.log 2>&1
timeout 400 python bench.py > gpurun_out/bench.json 2> gpurun_out/bench.err
timeout 300 ncu --set full --import-source on --clock-control none -k regex:k_tile -s 2 -c 1 -f -o gpurun_out/sb_full python tools/profile_frame.py --reps 1 > gpurun_out/ncu1.log 2>&1
tail -3 gpurun_out/gpu_tests.log
