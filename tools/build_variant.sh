#!/bin/bash
# build a diagnostic / A-B variant of the library: tools/build_variant.sh NAME "-DFLAG=1 ..." -> libstarsim_NAME.so
cd "$(dirname "$0")/.."
STARSIM_NVCC_EXTRA="$2" python -c "from paper_conf_ipps_lizzh12_b200 import _build; _build.build(force=True)" && \
  cp paper_conf_ipps_lizzh12_b200/libstarsim.so paper_conf_ipps_lizzh12_b200/libstarsim_$1.so
python -c "from paper_conf_ipps_lizzh12_b200 import _build; _build.build()"
