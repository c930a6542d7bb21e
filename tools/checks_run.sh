#!/bin/bash
# The GPU parity tests on a -DSTARSIM_CHECKS build (device-side bounds / invariant checks that trap; compute-sanitizer
# is closed on this pool): every check that fires fails the test that launched the kernel.
export STARSIM_NVCC_EXTRA="-DSTARSIM_CHECKS"
python -c "import __graft_entry__ as g; g.build()" > gpurun_out/build_checks.log 2>&1 || { tail gpurun_out/build_checks.log; exit 1; }
cat paper_conf_ipps_lizzh12_b200/libstarsim.so.flags > gpurun_out/checks_flags.txt
timeout 1500 python -m pytest tests -m gpu -q -x ${CHECKK:+-k "$CHECKK"} > gpurun_out/checks_tests.log 2>&1
tail -3 gpurun_out/checks_tests.log
