#!/bin/bash
# Build A/B variants of libbzk.so (compile-time knobs) next to the main library:
#   bash scripts/build_variants.sh NAME "NVCC FLAGS" [NAME "FLAGS"] ...
# -> paper_conf_asplos_lucw0cz25_b200/libbzk_NAME.so (use with BZK_LIB=...)
set -e
cd "$(dirname "$0")/.."
while [ $# -ge 2 ]; do
  name=$1; flags=$2; shift 2
  BZK_BUILD_DIR=/tmp/bzk_build_$name BZK_LIB_OUT=paper_conf_asplos_lucw0cz25_b200/libbzk_$name.so \
    BZK_NVCC_EXTRA="$flags" python -m paper_conf_asplos_lucw0cz25_b200.build --force &
done
wait
