#!/bin/bash
# A/B of one layer-pass GEMM under plan-option variants (tools/pass_time.py, CUDA events, warm),
# and of the filter-gradient split count on the -DGLP_DIAG build (GLP_DEBUG_SPLITS).  The round-2
# decisions recorded in DESIGN.md §7/§14 came from runs of this form, e.g.
#   PASS=caffenet_conv3:bwd_data WL=4 OPTS="'{}' '{\"tile_units\":6}'"   (tile model threshold)
#   PASS=lenet_conv1:bwd_filter WL=1 SPLITS="72 128 144"                  (small-filter splits)
cd "$(dirname "$0")/.."
MATH=${MATH:-fp32}
if [ -n "$OPTS" ]; then eval "WL=${WL:-4} python tools/pass_time.py $PASS $MATH $OPTS"; fi
if [ -n "$SPLITS" ]; then
  python -c "from paper_conf_icpp_futhys18_b200 import _build; _build.build(diag=True)"
  for S in $SPLITS; do
    echo "splits $S"
    GLP_LIB=$PWD/paper_conf_icpp_futhys18_b200/libglp_diag.so GLP_DEBUG_SPLITS=$S WL=${WL:-4} \
      python tools/pass_time.py $PASS $MATH '{}' 2>&1 | tail -1
  done
fi
