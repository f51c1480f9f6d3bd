#!/usr/bin/env bash
# SASS inspection build of one translation unit for one read width (no GPU needed):
#   scripts/sass_dev.sh partition_scatter.cu 4 scatter_table_kernel<4, true, false, 4>
# prints ptxas resource usage and writes /tmp/<unit>.sass (cuobjdump of the cubin)
set -eu
U=$1; W=${2:-4}
cd "$(dirname "$0")/../paper_conf_ipps_goswamilsp18_b200/csrc"
nvcc -O3 -std=c++17 -lineinfo -gencode arch=compute_100a,code=sm_100a -I ../../include \
     -DLSG_DEV_ONLY_W=$W -Xptxas -v -cubin -o /tmp/${U%.cu}.cubin $U 2>&1 | grep -E "Compiling|registers|spill" | paste - - - | sed 's/ptxas info    ://g' | cut -c1-260
cuobjdump -sass /tmp/${U%.cu}.cubin > /tmp/${U%.cu}.sass
