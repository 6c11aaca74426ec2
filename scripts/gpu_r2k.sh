cd "$(dirname "$0")/.."
for S in 36 72 96 128 144 192 288; do echo "splits $S"; GLP_LIB=$PWD/paper_conf_icpp_futhys18_b200/libglp_diag.so GLP_DEBUG_SPLITS=$S WL=1 python tools/pass_time.py lenet_conv1:bwd_filter fp32 '{}' 2>&1 | tail -1; done
for S in 8 16 32 64; do echo "splits $S"; GLP_LIB=$PWD/paper_conf_icpp_futhys18_b200/libglp_diag.so GLP_DEBUG_SPLITS=$S WL=2 python tools/pass_time.py lenet_conv2:bwd_filter fp32 '{}' 2>&1 | tail -1; done
