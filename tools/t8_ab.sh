#!/bin/bash
# same-box A/B of k_tile8 diagnostic builds at T (tile-kernel time from the library's per-kernel events)
cd "$(dirname "$0")/.."
build() {  # name, extra flags
  STARSIM_NVCC_EXTRA="$2" python -c "from paper_conf_ipps_lizzh12_b200 import _build; _build.build(force=True)" && \
    cp paper_conf_ipps_lizzh12_b200/libstarsim.so paper_conf_ipps_lizzh12_b200/libstarsim_$1.so
}
for v in "$@"; do
  name=${v%%=*}; flags=${v#*=}; [ "$name" = "$v" ] && flags=""
  build "$name" "$flags" > /dev/null 2>&1 || echo "build $name failed"
done
python -c "from paper_conf_ipps_lizzh12_b200 import _build; _build.build(force=True)" > /dev/null 2>&1
for v in "$@"; do
  name=${v%%=*}
  STARSIM_LIB=paper_conf_ipps_lizzh12_b200/libstarsim_$name.so timeout 300 python tools/ab_kern.py --config T --mode t8 | sed "s/^/$name /"
done
