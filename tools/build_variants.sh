#!/bin/bash
# Build experimental libsssp variants: tools/build_variants.sh "NAME:-DFLAG=.. -DFLAG2=.." ...
# Output: paper_conf_icppw_zhangczsdhay23_b200/libsssp_NAME.so (select with SSSP_LIB=...)
R=/root/repo
[ -n "$GRAFT_REPO_ROOT" ] && R=$GRAFT_REPO_ROOT
S=$R/paper_conf_icppw_zhangczsdhay23_b200/csrc/sssp_api.cu
for spec in "$@"; do
  name=${spec%%:*}; flags=${spec#*:}
  ( nvcc -gencode arch=compute_100a,code=sm_100a -O3 -lineinfo -std=c++17 -Xcompiler -fPIC -shared \
      $flags -Xptxas -v $S -o $R/paper_conf_icppw_zhangczsdhay23_b200/libsssp_$name.so 2>&1 \
      | grep -E "error|k_delta_stepILb0ELb1" -A2 | grep -E "error|registers|spill" | head -3 | sed "s/^/[$name] /" ) &
done
wait
