#!/bin/bash
# Build a variant of the library with extra nvcc defines into build_variants/<name>.so:
#   tools/build_variant.sh <name> -DFOO=1 ...
set -e
mkdir -p build_variants
name=$1; shift
FLB_LIB_PATH=build_variants/$name.so FLB_NVCC_EXTRA="$*" python paper_conf_icde_zeng0fcpcwg23_b200/build.py --force
