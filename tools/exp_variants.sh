#!/bin/bash
# Build experiment variants of libchecl.so under exp_libs/<name>/ (not shipped).
set -e
cd "$(dirname "$0")/.."
build() { name=$1; shift; mkdir -p exp_libs/$name; CHECL_LIB_OUT=$PWD/exp_libs/$name/libchecl.so CHECL_EXTRA_FLAGS="$*" python -m paper_conf_ipps_takizawakskk11_b200.build > /dev/null; echo built $name; }
for spec in "$@"; do name=${spec%%:*}; flags=${spec#*:}; [ "$flags" = "$spec" ] && flags=""; build $name ${flags//,/ }; done
