cd /root/repo
python tools/pass_time.py caffenet_conv1:bwd_filter fp32 '{}' '{"wgrad_tile_n":128}' '{"wgrad_tile_n":128,"max_kblocks_per_stage":1}' '{"max_kblocks_per_stage":1}' '{"max_kblocks_per_stage":2}'
python tools/pass_time.py caffenet_conv1:fwd fp32 '{}' '{"cta_pairs":0}' '{"max_kblocks_per_stage":1}' '{"max_kblocks_per_stage":2}'
python tools/pass_time.py caffenet_conv2:fwd fp32 '{}' '{"max_kblocks_per_stage":1}' '{"max_kblocks_per_stage":2}'
python tools/pass_time.py caffenet_conv2:bwd_data fp32 '{}' '{"max_kblocks_per_stage":1}'
python tools/pass_time.py caffenet_conv3:bwd_data fp32 '{}' '{"max_kblocks_per_stage":1}' '{"max_kblocks_per_stage":2}'
