#!/bin/bash
# Experimental library build with extra nvcc flags: tools/build_variant.sh NAME [flags...]
# -> build/lib_NAME.so (with its own patch cubin build/NAME.cubin); run with SWB_LIB=build/lib_NAME.so
set -e
name=$1; shift
cd "$(dirname "$0")/.."
mkdir -p build
F="-gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17"
nvcc $F "$@" -cubin -o build/$name.cubin paper_conf_ipps_sandesm11_b200/csrc/sw_fill16_patch.cu
python -c "import sys; sys.path.insert(0,'.'); from paper_conf_ipps_sandesm11_b200 import build as b; print(b.check_patch_sites('build/$name.cubin'))"
nvcc $F "$@" -Xcompiler -fPIC -shared -DSWB_PATCH_CUBIN="\"$PWD/build/$name.cubin\"" -o build/lib_$name.so paper_conf_ipps_sandesm11_b200/csrc/sw_api.cu
